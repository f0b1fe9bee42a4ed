timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputests.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --check > gpurun_out/bench.log 2>&1
bash tools/configs.sh gpurun_out/configs.jsonl
MSM_BENCH_SHARE_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --log2n 22 --check --steps 2 --no-cpu-baseline > gpurun_out/share2_default.log 2>&1
OUT=gpurun_out/prof_final KERNELS="k_accumulate_sync k_s3_part1 k_s3_part2 k_s3_part3" bash tools/profile_round.sh

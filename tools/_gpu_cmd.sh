timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --check > gpurun_out/bench.log 2>&1
for sp in buckets points; do
  MSM_BENCH_SHARE_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --log2n 22 --split $sp --check --steps 2 --no-cpu-baseline > gpurun_out/share2_$sp.log 2>&1
done
for so in 1 3; do timeout 600 python bench.py --log2n 24 --sort $so --steps 3 --no-e2e --no-cpu-baseline --check 2>/dev/null | tail -1 >> gpurun_out/sort_ablation.jsonl; done

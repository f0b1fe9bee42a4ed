timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --check > gpurun_out/bench.log 2>&1
python tools/ab.py --log2n 24 base pf2 > gpurun_out/ab_pf2.jsonl 2>&1
python tools/ab.py --log2n 26 --steps 2 base pf2 >> gpurun_out/ab_pf2.jsonl 2>&1
OUT=gpurun_out/prof_sort NOLAUNCH=1 KERNELS="k_s3_count1 k_s3_part1 k_s3_part2 k_s3_part3" bash tools/profile_round.sh
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_accumulate -s 3 -c 1 -o gpurun_out/acc_src -f python bench.py --log2n 22 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/acc_src.log 2>&1
ncu -i gpurun_out/acc_src.ncu-rep --page source --csv --print-source sass > gpurun_out/acc_src_sass.csv 2>&1
gzip -f gpurun_out/acc_src_sass.csv
rm -f gpurun_out/acc_src.ncu-rep

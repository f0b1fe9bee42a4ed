mkdir -p gpurun_out/accsrc
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_accumulate_sync -s 3 -c 1 -o gpurun_out/accsrc/acc -f python bench.py --log2n 22 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/accsrc/ncu.log 2>&1
ncu -i gpurun_out/accsrc/acc.ncu-rep --page source --csv --print-source sass > gpurun_out/accsrc/src.csv 2>/dev/null
gzip -f gpurun_out/accsrc/src.csv; rm -f gpurun_out/accsrc/acc.ncu-rep; ls -la gpurun_out/accsrc

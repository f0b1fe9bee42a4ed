mkdir -p gpurun_out/s4
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_s4 -c 3 -o gpurun_out/s4/s4full -f python bench.py --sort 4 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/s4/ncu.log 2>&1; tail -3 gpurun_out/s4/ncu.log

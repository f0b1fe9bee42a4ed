mkdir -p gpurun_out/c1src
export MSM_LIB=$PWD/build_dev/libmsm_dev.so
for k in k_accumulate_sync k_bucket_segments; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/c1src/$k -f python bench.py --curve bn254 --log2n 10 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-check > gpurun_out/c1src/$k.log 2>&1
done
ls -la gpurun_out/c1src

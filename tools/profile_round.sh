#!/bin/bash
# ncu evidence for one round (run under gpurun, one GPU):
#   launch list of the bench step (cold-cache, serialised) + full-set captures of the
#   dominant kernels.  Output under gpurun_out/prof/.
cd "$(dirname "$0")/.."
o=${OUT:-gpurun_out/prof}; mkdir -p $o
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-check ${BENCH_ARGS}"
[ -z "$NOLAUNCH" ] && timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv --log-file $o/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-check > $o/launches.log 2>&1
for k in ${KERNELS:-k_accumulate k_bucket_segments k_s3_scatter}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o $o/$k -f $B > $o/$k.log 2>&1
  ncu -i $o/$k.ncu-rep --page raw --csv > $o/${k}_raw.csv 2>/dev/null
  ncu -i $o/$k.ncu-rep --page details --csv > $o/${k}_details.csv 2>/dev/null
  rm -f $o/$k.ncu-rep  # reports are tens of MB; gpurun copies back <= 64 MiB
done

#!/bin/bash
# Round-2 GPU evidence (one GPU, under gpurun): all BASELINE configs + the C2 c sweep
# (each with the closed-form check), the ncu launch list of the C4 step, and full-set ncu
# captures of the dominant kernels.  Output under gpurun_out/r02/.
cd "$(dirname "$0")/.."
o=gpurun_out/r02; mkdir -p $o
bash tools/configs.sh $o/configs.jsonl
OUT=$o/prof KERNELS="k_accumulate_sync k_bucket_segments k_s3_part1 k_s3_part2 k_s3_part3" bash tools/profile_round.sh
ls -la $o $o/prof

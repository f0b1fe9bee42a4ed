MSM_LIB=variants/libmsm_smem.so timeout 900 python -m pytest tests -m gpu -x -q -k "bls12_381" > gpurun_out/smem_tests.log 2>&1
python tools/ab.py --log2n 24 base smem > gpurun_out/ab_smem.jsonl 2>&1
python tools/ab.py --log2n 26 --steps 2 base smem >> gpurun_out/ab_smem.jsonl 2>&1

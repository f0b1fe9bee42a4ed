MSM_LIB=variants/libmsm_pf3.so timeout 1200 python -m pytest tests -m gpu -q -k "bls12_381 or bn254 or large or oversized or degenerate" > gpurun_out/pf3_tests.log 2>&1
python tools/ab.py --log2n 24 base sortopt pf3 > gpurun_out/ab_pf3.jsonl 2>&1
python tools/ab.py --log2n 26 --steps 3 base sortopt pf3 >> gpurun_out/ab_pf3.jsonl 2>&1

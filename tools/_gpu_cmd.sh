timeout 900 python tools/ab.py --log2n 24 accsync sync384 > gpurun_out/ab_sync384.jsonl 2>&1
timeout 900 python tools/ab.py --log2n 26 --steps 3 accsync sync384 >> gpurun_out/ab_sync384.jsonl 2>&1

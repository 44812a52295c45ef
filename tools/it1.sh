timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "random or c2_full or t0 or per_pc" 2>&1 | tail -3
bash tools/ab.sh "c2:15,2 c3:15" cur r0 r1 lg12 lg10 2>&1

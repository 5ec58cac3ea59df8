#!/bin/bash
# Round-2 GPU check: -m gpu suite, smoke, full-size parity (C3/C4/C5), default bench line.
O=gpurun_out/r2check; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
( time timeout 2400 python -m pytest tests -m gpu -x -q ) > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 600 python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
( time timeout 1800 python tools/parity_full.py --configs ${CONFIGS:-C3,C4,C5} --out $O ) > $O/parity.log 2>&1; echo "parity rc=$?"; grep -o '"config": "C[0-9]"\|"exact": [a-z]*\|"max_rel": [0-9.e-]*\|"l1": [0-9.e-]*' $O/parity.log
timeout 900 python bench.py > $O/bench.log 2>&1; echo "bench rc=$?"; tail -1 $O/bench.log | cut -c1-600

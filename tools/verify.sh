#!/bin/bash
# round-end check: GPU tests, smoke, default bench line (C2)
O=gpurun_out/verify; mkdir -p $O
make -j4 all > $O/build.log 2>&1; echo "build rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"; tail -c 1500 $O/bench_C2.json

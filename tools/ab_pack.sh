#!/bin/bash
# A/B: packed (count, degree) tile scan in the fused dense tile only (pack) vs also in the two-walk pass 2 (pack2); GPU tests, smoke
O=gpurun_out/pack2; mkdir -p $O
V=build/variants
timeout 900 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python tools/kbench.py --config C2 --alg bfs --part degree --runs 16 --libs $V/libgum_pack.so,$V/libgum_pack2.so > $O/kb_c2.txt 2>&1; cat $O/kb_c2.txt

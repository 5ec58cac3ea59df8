#!/bin/bash
# A/B: filter L1 prefetch one tile ahead (GUM_FILTER_PREFETCH) and filter CTAs per SM via GUM_FILTER_MINB builds
O=gpurun_out/pf; mkdir -p $O
V=build/variants
for r in 1 2; do
  GUM_FILTER_PREFETCH=0 timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 16 --libs $V/libgum_pf.so | sed 's/^/nopf /'
  timeout 600 python tools/kbench.py --config C2 --alg bfs --part degree --runs 16 --libs $V/libgum_pf.so,$V/libgum_pf_m5.so,$V/libgum_pf_m6.so
done > $O/kb_c2.txt 2>&1; cat $O/kb_c2.txt
for L in pf pf_m6; do GUM_FILTER_PREFETCH=0 timeout 600 python tools/kbench.py --config C4 --alg wcc --runs 4 --libs $V/libgum_$L.so | sed 's/^/nopf /'; timeout 600 python tools/kbench.py --config C4 --alg wcc --runs 4 --libs $V/libgum_$L.so; done > $O/kb_c4.txt 2>&1; cat $O/kb_c4.txt
timeout 900 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log

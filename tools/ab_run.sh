O=gpurun_out/ab2; mkdir -p $O
./tools/plantest/plantest_old > $O/plantest_old.txt 2>&1; echo "old rc=$?"; tail -1 $O/plantest_old.txt
./tools/plantest/plantest > $O/plantest_new.txt 2>&1; echo "new rc=$?"; tail -1 $O/plantest_new.txt
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "planned or cost_model" > $O/pytest_plan.txt 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_plan.txt
timeout 300 python tools/iter_trace.py --config C2 --alg bfs --part degree --runs 5 > $O/iter_C2.txt 2>&1; cat $O/iter_C2.txt
timeout 900 python tools/ablation.py --table4 --scale 22 --grid 2048 --workers 8 --delta 1024 --out $O/abl_table4.json > $O/abl_table4.txt 2>&1; echo "table4 rc=$?"; cat $O/abl_table4.txt

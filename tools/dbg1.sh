O=gpurun_out/dbg1; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_dpr.py -q > $O/dpr.log 2>&1; echo "dpr rc=$?"; tail -3 $O/dpr.log; grep -E "^E  " $O/dpr.log | head -20

O=gpurun_out/dbg1; mkdir -p $O
timeout 1800 python -m pytest tests/test_gpu_units.py tests/test_gpu_mp.py -q --maxfail=20 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log; grep -E "^FAILED|^E   .*mismatch" $O/pytest.log | head -20

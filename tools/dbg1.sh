O=gpurun_out/dbg1; mkdir -p $O
( time timeout 2400 python -m pytest tests -m gpu -q --maxfail=30 ) > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -4 $O/pytest.log; grep -E "^FAILED" $O/pytest.log | head -30

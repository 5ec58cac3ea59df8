O=gpurun_out/ab15; mkdir -p $O
timeout 400 python tools/dbg_mp_iters.py > $O/mp.txt 2>&1; echo "mp rc=$?"; grep -v Warn $O/mp.txt | tail -16
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.txt 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.txt

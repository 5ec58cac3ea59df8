O=gpurun_out/ab20; mkdir -p $O
( time timeout 1800 python -m pytest tests -m gpu -q ) > $O/pytest.txt 2>&1; echo "pytest rc=$?"; grep passed $O/pytest.txt | tail -1
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --split --out $O/abl_osteal_split.json > $O/abl_osteal_split.txt 2>&1; cat $O/abl_osteal_split.txt
timeout 400 python tools/dbg_mp_iters.py > $O/mp.txt 2>&1; grep -v Warn $O/mp.txt | tail -8

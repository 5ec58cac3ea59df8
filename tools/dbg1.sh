O=gpurun_out/dbg1; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/t.log 2>&1; echo "tests rc=$?"; tail -2 $O/t.log | head -1; grep -E "^FAILED" $O/t.log | head -5
timeout 900 python tools/ablation.py --table4 --scale 22 --grid 2048 --workers 8 --delta 1024 --out $O/abl_table4.json > $O/abl_table4.txt 2>&1; cat $O/abl_table4.txt
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --split --out $O/abl_osteal_split.json > $O/abl_osteal_split.txt 2>&1; cat $O/abl_osteal_split.txt

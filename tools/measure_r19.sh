#!/bin/bash
O=gpurun_out/r19; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
python tools/profile_run.py --rmat 22 --noscramble --gpus 8 --runs 3 --alg bfs > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-300
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal.txt 2>&1; cat $O/abl_fsteal.txt
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --split --out $O/abl_fsteal_split.json > $O/abl_fsteal_split.txt 2>&1; cat $O/abl_fsteal_split.txt
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal.txt 2>&1; cat $O/abl_osteal.txt

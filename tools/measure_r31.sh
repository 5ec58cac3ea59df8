#!/bin/bash
O=gpurun_out/r31; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py tests/test_gpu_mp.py -m gpu -q -x -k "tail or grid or near_far or hand or virtual or forced or mp" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
python tools/profile_run.py --grid 2048 --alg sssp --gpus 8 --delta 1024 --osteal-threshold 4096 --runs 2 > $O/prof.txt 2>&1; echo "P8 grid $(tail -1 $O/prof.txt | cut -c1-220)"
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal.txt 2>&1; cat $O/abl_osteal.txt
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal.txt 2>&1; cat $O/abl_fsteal.txt

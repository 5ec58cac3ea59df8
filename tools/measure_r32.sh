#!/bin/bash
O=gpurun_out/r32; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 3 -c 1 -o $O/adv_C2_bfs python tools/profile_run.py --runs 1 --config C2 --alg bfs --part degree > /dev/null 2>&1; echo "rc=$?"

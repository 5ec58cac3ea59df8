#!/bin/bash
O=gpurun_out/r29; mkdir -p $O
for lib in build/variants/libgum_old.so paper_conf_icde_menggltyz23_b200/libgum.so; do
  GUM_LIB=$lib python tools/profile_run.py --grid 2048 --alg sssp --gpus 8 --delta 1024 --osteal-threshold 4096 --runs 2 > $O/prof.txt 2>&1; echo "$lib"; tail -2 $O/prof.txt | cut -c1-420
done

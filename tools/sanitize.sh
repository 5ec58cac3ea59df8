#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over every algorithm on RMAT-12, in four launch modes
# (one worker, 4 virtual workers, 4 split launch units = the device-resident multi-unit loop, 2 processes
# with CUDA IPC). Logs: $O/<tool>_<mode>.log; summary: $O/summary.txt.
O=${O:-gpurun_out/sanitize}; mkdir -p $O
: > $O/summary.txt
for tool in memcheck racecheck synccheck; do
  for mode in single virtual4 split4 mp2; do
    log=$O/${tool}_${mode}.log
    if [ $mode = mp2 ]; then
      timeout 600 compute-sanitizer --tool $tool --target-processes all --print-limit 50 \
        python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
        tools/sanitize_case.py mp2 > $log 2>&1
    else
      timeout 600 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_case.py $mode > $log 2>&1
    fi
    rc=$?
    echo "$tool $mode rc=$rc $(grep -h 'ERROR SUMMARY' $log | tr '\n' ' ') $(grep -h 'SANITIZE_CASE' $log | tr '\n' ' ')" | tee -a $O/summary.txt
  done
done

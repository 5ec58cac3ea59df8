O=gpurun_out/dbg1; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -k "split_units_multi_device_path or planned_fsteal or pr_pull or mirrors" > $O/pytest2.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest2.log; grep -E "^FAILED" $O/pytest2.log | head

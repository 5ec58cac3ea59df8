O=gpurun_out/ab7; mkdir -p $O
V=build/variants
timeout 900 python tools/kbench.py --config C5 --alg pr --part degree --runs 3 --libs $V/libgum_pullnopad.so,$V/libgum_pullpad.so > $O/pull_pad_C5.txt 2>&1; cat $O/pull_pad_C5.txt
timeout 900 python -m pytest tests -m gpu -x -q -k "pr or pull" > $O/pytest.txt 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.txt

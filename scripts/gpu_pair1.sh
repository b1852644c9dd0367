cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "two_layer or toy or geometry" > gpurun_out/pair_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/pair_tests.log
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 > gpurun_out/pair_gpt.log 2>&1
echo "gpt rc=$?" >> gpurun_out/pair_gpt.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "fuzz" > gpurun_out/pair_fuzz.log 2>&1
echo "fuzz rc=$?" >> gpurun_out/pair_fuzz.log

cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "two_layer or toy or geometry or fuzz" > gpurun_out/pair_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/pair_tests.log
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 > gpurun_out/pair_ab.log 2>&1
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 >> gpurun_out/pair_ab.log 2>&1

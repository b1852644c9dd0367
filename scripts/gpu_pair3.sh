cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "two_layer or toy or geometry or fuzz" > gpurun_out/pair_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/pair_tests.log
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 > gpurun_out/pair_gpt.log 2>&1
echo "gpt rc=$?" >> gpurun_out/pair_gpt.log
MADPIPE_KERNEL=pair timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_step -s 60 -c 1 -o gpurun_out/prof_pair python scripts/exp_batch_l2.py gpt 0 > gpurun_out/ncu_pair.log 2>&1

cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "two_layer or toy or geometry or fuzz" > gpurun_out/pair_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/pair_tests.log
MADPIPE_PAIR_OVERLAP=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "two_layer or toy or fuzz" >> gpurun_out/pair_tests.log 2>&1
echo "tests overlap rc=$?" >> gpurun_out/pair_tests.log
MADPIPE_PROF=1 MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 > gpurun_out/pair_prof.log 2>&1
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 >> gpurun_out/pair_prof.log 2>&1
MADPIPE_KERNEL=pair MADPIPE_PAIR_OVERLAP=1 timeout 300 python scripts/exp_batch_l2.py gpt 0 >> gpurun_out/pair_prof.log 2>&1
MADPIPE_KERNEL=pair timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_pair.csv python scripts/exp_batch_l2.py gpt 0 > gpurun_out/ncu_pair_launch.log 2>&1

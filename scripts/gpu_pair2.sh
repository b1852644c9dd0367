cd $GRAFT_REPO_ROOT
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py gpt 0 > gpurun_out/pair_gpt.log 2>&1
MADPIPE_KERNEL=persist timeout 300 python scripts/exp_batch_l2.py gpt 0 >> gpurun_out/pair_gpt.log 2>&1
MADPIPE_KERNEL=pair timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_step -s 60 -c 1 -o gpurun_out/prof_pair python scripts/exp_batch_l2.py gpt 0 > gpurun_out/ncu_pair.log 2>&1
MADPIPE_KERNEL=pair timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_pair.csv python scripts/exp_batch_l2.py gpt 0 > gpurun_out/ncu_pair_launch.log 2>&1

cd $GRAFT_REPO_ROOT
for r in 4 8 16 24; do
MADPIPE_KERNEL=pair MADPIPE_PAIR_ROUND=$r timeout 300 python scripts/exp_batch_l2.py gpt 0 >> gpurun_out/pair_round.log 2>&1
done
for k in resnet50 inception_v3 vgg19; do
MADPIPE_KERNEL=pair timeout 300 python scripts/exp_batch_l2.py $k 0 >> gpurun_out/pair_cnn.log 2>&1
MADPIPE_KERNEL=persist timeout 300 python scripts/exp_batch_l2.py $k 0 >> gpurun_out/pair_cnn.log 2>&1
timeout 300 python scripts/exp_batch_l2.py $k 0 >> gpurun_out/pair_cnn.log 2>&1
done

cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1
timeout 900 python bench.py --config gpt --steps 3 --warmup 3 > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu --force-dist > gpurun_out/bench_gpt_dist.json 2> gpurun_out/bench_gpt_dist.err
for c in resnet50 inception_v3 vgg19; do timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
timeout 600 python scripts/fig6_sweep.py --out gpurun_out/fig6_resnet50.md > gpurun_out/fig6.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gpt.csv python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch.log 2>&1
timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:step_persist -s 300 -c 40 --csv --log-file gpurun_out/traffic_gpt.csv python bench.py --config gpt --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_traffic.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:step_persist -s 500 -c 1 -o gpurun_out/prof_step python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1
echo done

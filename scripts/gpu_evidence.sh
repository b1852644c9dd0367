# GPU evidence (run through gpurun from the repo root; profiles/r02b_* came from STAGES="test bench prof").  STAGES selects parts:
#   test   : build, smoke(), pytest -m gpu
#   bench  : bench.py gpt (N=1), gpt through the N-GPU code path (torchrun world 1, ctx-owned
#            NCCL communicator), batch config, CNN configs
#   prof   : ncu launch list of the bench, DRAM traffic of every step launch of one sweep,
#            one --set full capture of the step kernel
#   san    : compute-sanitizer memcheck / racecheck / synccheck of the small-case script, per part
#   fp64   : tools/fp64peak (measured FP64 DADD / DFMA / relaxation throughput)
#   batchprof : per-batch timing of the C5 batch config (MADPIPE_PROF=1)
#   gptbench  : only the GPT bench line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
STAGES="${STAGES:-test bench}"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
if [[ $STAGES == *test* ]]; then
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
  timeout 2400 python -m pytest tests -m gpu -q --durations=15 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
fi
if [[ $STAGES == *gptbench* || $STAGES == *bench* ]]; then
  timeout 900 python bench.py --config gpt --steps 3 --warmup 3 > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
fi
if [[ $STAGES == *fp64* ]]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fp64peak tools/fp64peak.cu && ./tools/fp64peak > gpurun_out/fp64_peak.json 2>&1
fi
if [[ $STAGES == *batchprof* ]]; then
  MADPIPE_PROF=1 timeout 900 python bench.py --config batch --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/batchprof.json 2> gpurun_out/batchprof.err
fi
if [[ $STAGES == *" bench"* || $STAGES == bench* ]]; then
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu --force-dist > gpurun_out/bench_gpt_torchrun_world1.json 2> gpurun_out/bench_gpt_torchrun_world1.err
  timeout 900 python bench.py --config batch --steps 3 --warmup 3 > gpurun_out/bench_batch.json 2> gpurun_out/bench_batch.err
  for c in resnet50 inception_v3 vgg19; do timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
fi
if [[ $STAGES == *prof* ]]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gpt.csv python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch.log 2>&1
  timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:pair_step --csv --log-file gpurun_out/traffic_gpt.csv python scripts/gpt_one_sweep.py gpurun_out/one_sweep.json > gpurun_out/ncu_traffic.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:pair_step -s 300 -c 1 -o gpurun_out/prof_pair_step python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1
fi
if [[ $STAGES == *san* ]]; then
  for tool in memcheck racecheck synccheck; do
    for part in base pair persist literal; do
      timeout 1500 compute-sanitizer --tool $tool --print-limit 30 python scripts/sanitize_small.py $part > gpurun_out/sanitize_${tool}_$part.log 2>&1
      echo "$tool $part rc=$?" >> gpurun_out/sanitize_${tool}_$part.log
    done
  done
fi
echo done

cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
STAGES="test" bash scripts/gpu_r02.sh
D=paper_conf_ipps_beaumontes22_b200
for i in 1 2; do
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/ab_base_$i.json 2>/dev/null
  MADPIPE_LIB=$PWD/$D/libmadpipe_qatomic.so timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/ab_qatomic_$i.json 2>/dev/null
done
timeout 900 python bench.py --config batch --steps 3 --warmup 3 > gpurun_out/bench_batch.json 2> gpurun_out/bench_batch.err
MADPIPE_PROF=1 timeout 900 python bench.py --config batch --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/batchprof.json 2> gpurun_out/batchprof.err
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o tools/racecheck_repro tools/racecheck_repro.cu
./tools/racecheck_repro > gpurun_out/racecheck_repro_plain.log 2>&1
timeout 300 compute-sanitizer --tool racecheck --print-limit 20 ./tools/racecheck_repro > gpurun_out/racecheck_repro.log 2>&1
for tool in racecheck synccheck; do
  for part in base pair persist literal; do
    timeout 1500 compute-sanitizer --tool $tool --print-limit 30 python scripts/sanitize_small.py $part > gpurun_out/sanitize_${tool}_$part.log 2>&1
    echo "$tool $part rc=$?" >> gpurun_out/sanitize_${tool}_$part.log
  done
done
MADPIPE_LIB=$PWD/$D/libmadpipe_qatomic.so timeout 1500 compute-sanitizer --tool racecheck --print-limit 30 python scripts/sanitize_small.py pair > gpurun_out/sanitize_racecheck_pair_qatomic.log 2>&1
echo done

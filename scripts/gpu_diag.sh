# Step-kernel bound diagnostics (MADPIPE_REPLAY on the MP_DIAG=1 build, scripts/build_variants.py diag):
# the GPT pass-64 step launch re-run on its real lists with the relaxation and/or the copies removed.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
D=paper_conf_ipps_beaumontes22_b200
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_throttle_reasons.active --format=csv > gpurun_out/diag_smi.txt
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/diag_bench.json 2> gpurun_out/diag_bench.err
for p in ${PASSES:-64}; do for dg in 0 1 2 3; do
  MADPIPE_REPLAY=$p,10,$dg MADPIPE_LIB=$PWD/$D/libmadpipe_diag.so timeout 300 python scripts/gpt_one_sweep.py /tmp/x.json 2>&1 | grep replay > gpurun_out/diag_r${p}_$dg.txt
done; done
echo done

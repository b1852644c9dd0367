# Same-box A/B: pair-path parity tests on the default build, then the GPT bench for each
# library in VARS (default = libmadpipe.so; others = libmadpipe_<v>.so, e.g. r2 = the last
# committed kernel built from a worktree) and each producer round size in ROUNDS, two
# interleaved rounds; MADPIPE_PROF counters of the default build; the pass-64 step replay
# with the relaxation / copies removed (diag build).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
D=paper_conf_ipps_beaumontes22_b200
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_throttle_reasons.active --format=csv > gpurun_out/ab_smi.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "${PTEST:-two_layer or mixed or toy or counters or comm_heavy or geometry}" > gpurun_out/ab_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab_pytest.log
tail -3 gpurun_out/ab_pytest.log
for i in 1 2; do for v in ${VARS:-default r2}; do for rd in ${ROUNDS:-0}; do
  L=$PWD/$D/libmadpipe_$v.so; [ "$v" = default ] && L=$PWD/$D/libmadpipe.so
  E=""; [ "$rd" != 0 ] && E="MADPIPE_PAIR_ROUND=$rd"
  env $E MADPIPE_LIB=$L timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/ab_${v}_r${rd}_$i.json 2> gpurun_out/ab_${v}_r${rd}_$i.err
done; done; done
MADPIPE_PROF=1 timeout 300 python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e > gpurun_out/ab_prof.json 2> gpurun_out/ab_prof.err
if [ -f $D/libmadpipe_diag.so ]; then for dg in 0 1 2 3; do
  MADPIPE_REPLAY=64,10,$dg MADPIPE_LIB=$PWD/$D/libmadpipe_diag.so timeout 300 python scripts/gpt_one_sweep.py /tmp/x.json 2>&1 | grep replay > gpurun_out/ab_r64_$dg.txt
done; fi
echo done

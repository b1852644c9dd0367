# Same-box A/B of the pair kernel's producer round size (MADPIPE_PAIR_ROUND, read per launch) and
# consumer back-off variants (prebuilt by scripts/build_variants.py), GPT bench, two rounds.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
D=paper_conf_ipps_beaumontes22_b200
for i in 1 2; do
  for r in 8 10 12 14 16; do
    MADPIPE_PAIR_ROUND=$r timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/round${r}_$i.json 2>/dev/null
  done
  for v in poll0 poll100; do
    MADPIPE_LIB=$PWD/$D/libmadpipe_$v.so timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/var_${v}_$i.json 2>/dev/null
  done
done
echo done

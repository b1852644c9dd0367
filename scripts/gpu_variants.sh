# Same-box A/B of pair-kernel compile-time variants, each prebuilt as its own library
# (MADPIPE_DEFS=... MADPIPE_LIB=.../libmadpipe_<name>.so): parity tests of the pair path,
# then the GPT bench, two interleaved rounds.
cd $GRAFT_REPO_ROOT
D=paper_conf_ipps_beaumontes22_b200
VARS="${VARS:-base vb8}"
for v in $VARS; do
  echo "$v: $(cat $D/libmadpipe_$v.so.flags)" >> gpurun_out/var_flags.txt
  MADPIPE_LIB=$PWD/$D/libmadpipe_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "two_layer or mixed or toy or counters or comm_heavy or geometry" > gpurun_out/var_pytest_$v.log 2>&1; echo "rc=$?" >> gpurun_out/var_pytest_$v.log
done
for i in 1 2; do for v in $VARS; do
  MADPIPE_LIB=$PWD/$D/libmadpipe_$v.so timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/var_${v}_$i.json 2> gpurun_out/var_${v}_$i.err
done; done
echo done

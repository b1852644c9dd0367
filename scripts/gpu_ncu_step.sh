# ncu --set full (source-level) capture of one mid-sweep pair step launch, library MADPIPE_LIB (default libmadpipe.so).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
D=paper_conf_ipps_beaumontes22_b200
export MADPIPE_LIB=$PWD/$D/libmadpipe${V:+_$V}.so
python scripts/gpt_one_sweep.py /tmp/x.json > gpurun_out/ncuq_plain.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:${K:-pair_step_kernel} -s 64 -c 1 \
    -o gpurun_out/ncu_step${V:+_$V} python scripts/gpt_one_sweep.py /tmp/x.json > gpurun_out/ncuq_ncu.log 2>&1
echo rc=$?

# Q4.1 plan prefixes (scan only, + each probe, + group-by) at SF30 and SF100
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/abl
for sf in 30 100; do timeout 900 python scripts/ablate_q41.py $sf > gpurun_out/abl/q41_sf$sf.log 2>&1; echo SF$sf; cat gpurun_out/abl/q41_sf$sf.log; done

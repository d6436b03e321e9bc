cd $GRAFT_REPO_ROOT
O=gpurun_out/r02fin4; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -2 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 1500 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 200 $O/bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o $O/ssb_q41_sf100_jit python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > $O/ncu_q41.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o $O/ssb_q31_sf30_jit python scripts/profile_query.py --query ssb_q31 --sf 30 --reps 2 > $O/ncu_q31.log 2>&1
timeout 1200 python scripts/dist_emulate.py --query ssb_q41 --sf 100 --out $O/dist_emulate_q41.json > $O/dist_emulate.log 2>&1
ls $O

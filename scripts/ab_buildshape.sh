# A/B of the dimension-build kernels' shape (rows per thread x blocks per SM) through library
# variants built with -DHQ_BUILD_U / -DHQ_BUILD_MINB (HQ_LIB_PATH selects one)
cd $GRAFT_REPO_ROOT
for lib in paper_conf_sigmod_funkebnmt18_b200/libhq.so build/var/libhq_16_4.so build/var/libhq_4_8.so build/var/libhq_8_3.so; do
  echo "== $lib"
  for qs in "ssb_q41 100" "tpch_q3 30"; do set -- $qs
    HQ_LIB_PATH=$PWD/$lib python scripts/step_trace.py --query $1 --sf $2 2>&1 | grep -E 'build|rank|step 2' | sed 's/(anonymous namespace):://' | cut -c1-90
  done
done

cd $GRAFT_REPO_ROOT
for e in fused multipass oaat; do echo "== $e"; timeout 300 python scripts/profile_query.py --query ssb_q21 --sf 30 --reps 2 --exec $e 2>&1 | tail -1; done
for e in multipass oaat; do echo "== $e sf3"; timeout 300 python scripts/profile_query.py --query ssb_q21 --sf 3 --reps 2 --exec $e 2>&1 | tail -1; done
echo "== sanitizer multipass sf3"; timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python scripts/profile_query.py --query ssb_q21 --sf 3 --reps 1 --exec multipass 2>&1 | grep -v "^=========     " | head -30

# pack_embed: current (A) vs the r02prof kernel (B): parity tests on A, per-class times on both
cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_elementwise_r02prof.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/elementwise.cu \
  TESTK="embed or unpack or parity" BENCH=scripts/r02/bench_classes.py WL="c2 c3 c4" TAG=${TAG:-emb} \
  bash scripts/r02/ab_two.sh 2>&1 | grep -v '"us": 0'

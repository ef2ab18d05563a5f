cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-online}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
for ld in 0.5 1.0 2.0; do timeout 600 python bench.py --online --load $ld > $T/online_$ld.json 2> $T/online_$ld.err; echo online $ld rc $?; tail -2 $T/online_$ld.err; done
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $T/ref.json 2> $T/ref.err; echo ref rc $?

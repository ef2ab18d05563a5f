cd $GRAFT_REPO_ROOT; T=gpurun_out/fold; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 900 python -m pytest tests -m gpu -q -x -k "embed or parity or smoke" -p no:cacheprovider --timeout 300 > $T/pytest.log 2>&1; echo pytest rc $?; tail -2 $T/pytest.log
ENVS="TCB_EMB_FOLD=1|TCB_EMB_FOLD=0" WL="c3 c4" TAG=fold bash scripts/r02/env_sweep.sh 2>&1 | grep -E "env|embed|step"

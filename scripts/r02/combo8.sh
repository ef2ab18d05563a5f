cd $GRAFT_REPO_ROOT; T=gpurun_out/tail; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 900 python -m pytest tests -m gpu -q -x -k "linear_ln or parity or smoke" -p no:cacheprovider --timeout 300 > $T/pytest.log 2>&1; echo pytest rc $?; tail -2 $T/pytest.log
ENVS="TCB_LNG_TAIL=1|TCB_LNG_TAIL=0" WL="c2 c3" TAG=tail bash scripts/r02/env_sweep.sh

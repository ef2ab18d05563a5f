# quick A/B: kernel parity tests + bench per workload (per-class times)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { echo build failed; tail gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x --timeout 300 --timeout_method thread -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -3
for w in ${WORKLOADS:-c2 c3 c4 c5}; do
  timeout 300 python bench.py --steps 20 --warmup 5 --workload $w --no-cpu-baseline > gpurun_out/ab_$w.json 2> gpurun_out/ab_$w.err; echo bench $w rc $?
  python - $w <<'PY'
import json,sys; w=sys.argv[1]; d=json.load(open(f'gpurun_out/ab_{w}.json'))
print(w, round(d['value']/1e6,3), 'Mtok/s', round(d['ms_per_step'],3), 'ms', d['clocks']['sm_mhz'], d['clocks']['reasons'])
print('   ' + ' '.join(f"{k}={c['us_per_launch']:.1f}" for k,c in d['roofline']['classes'].items()))
PY
done

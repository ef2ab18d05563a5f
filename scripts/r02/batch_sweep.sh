# tokens/s and whole-step tensor fraction vs batch rows per GPU (bench.py --rows)
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-bsweep}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
for spec in ${SPECS:-c2:128 c2:256 c2:512 c2:1024 c3:32 c3:64 c3:128 c3:256 c5:64 c5:128 c5:256}; do
  w=${spec%%:*}; r=${spec##*:}
  timeout 600 python bench.py --workload $w --rows $r --steps 10 --warmup 3 --no-cpu-baseline > $T/${w}_${r}.json 2>$T/err_${w}_${r}.txt
  python - $w $r $T/${w}_${r}.json <<'PY' | tee -a $T/sweep.jsonl
import json, sys
w, r, f = sys.argv[1:]
try:
    d = json.loads([l for l in open(f) if l.startswith("{")][-1])
    print(json.dumps({"workload": w, "rows": int(r), "tokens_per_s": d["value"], "ms_per_step": d["ms_per_step"],
                      "tc_frac_whole_step": d["tc_frac_whole_step"], "clocks": d["clocks"]}))
except Exception as e:
    print(json.dumps({"workload": w, "rows": int(r), "error": str(e)}))
PY
done

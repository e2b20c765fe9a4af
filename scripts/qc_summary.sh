# Summarise gpurun_out/qc_* (pytest tail + one line per bench log)
tail -4 gpurun_out/qc_pytest.log
for f in gpurun_out/qc_bench*.log; do
  echo "== $f"
  grep '^{' "$f" | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); r=d.get('roofline') or {}
    print('%.4g'%d['value'], 'ms/step=%.4f'%d['ms_per_step'], str(r.get('kernel',''))[:50], r.get('frac'), d['config'].get('workload','')[:90])
"
  grep -v '^{' "$f" | tail -3
done

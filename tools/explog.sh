#!/bin/bash
# summarise gpurun_out/exp/*.log (experiment session logs)
for f in $(ls gpurun_out/exp/*.log | sort -t/ -k3 -n); do head -1 $f; grep -E "passed|failed|rc=|Error|error" $f | tail -3; grep '^{' $f | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); r=d.get('roofline') or {}; print('  value %.4g frac %s kernel_ms %s e2e %s'%(d['value'], r.get('frac'), r.get('kernel_ms'), (d.get('e2e') or {}).get('value')))"; done

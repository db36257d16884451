#!/bin/bash
O=gpurun_out/${TAG:-m6}; mkdir -p $O
GPL_DEBUG_TUNE=1 GPL_DEBUG_MODEL=1 timeout 2400 python -c "
import experiments, json
s = experiments.model_vs_autotune(qs=tuple('${QS:-Q9 Q5}'.split()), out='$O/model_vs_autotune_sf100.json')
print(json.dumps({k: v for k, v in s.items() if k != 'points'}))
for p in s['points']: print(p['query'], p['model_ms'], p['autotune_ms'], p['model_over_autotune'], p['model_shape'], p['autotune_shape'])
" > $O/model.log 2>&1; grep -v "^autotune" $O/model.log | grep -v "^apply_profile" | tail -8; grep "^apply_profile" $O/model.log | sort | uniq -c

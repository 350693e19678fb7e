python __graft_entry__.py build > /dev/null
CUSAN_DEBUG_TIMING=1 timeout 300 python tools/session_bench.py --config 5 --chunk 512 > gpurun_out/ses_seq_512.json 2>gpurun_out/ses_dbg_512.txt; python - <<'PY'
import json
d=json.load(open('gpurun_out/ses_seq_512.json'))
lines=open('gpurun_out/ses_dbg_512.txt').read().split('\n')
calls=[]; cur={}
for l in lines:
    if not l.startswith('cusan_session:'): continue
    parts=l.split(); cur[parts[1]]=float(parts[2])
    if parts[1]=='merge': calls.append(cur); cur={}
for i,(c,p) in enumerate(zip(calls,d['per_call'])):
    if p['seconds']*1e3-p['kernel_ms']>5: print(i, round(p['seconds']*1e3,1), c)
PY

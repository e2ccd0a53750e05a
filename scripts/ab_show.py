import json, sys
for l in open(sys.argv[1] if len(sys.argv) > 1 else 'gpurun_out/ab.json'):
    d = json.loads(l)
    ks = sorted(d['kernels'].items(), key=lambda x: -x[1]['ms_per_step'])[:7]
    print(d.get('variant', '-'), d['config']['workload'][:12], round(d['ms_per_step'], 2), {k: round(v['ms_per_step'], 2) for k, v in ks})

import json, sys
d = json.load(open(sys.argv[1] if len(sys.argv) > 1 else 'gpurun_out/bench.json'))
rf = d['roofline']
print('value', round(d['value']), 'GFLOP/s  ms', round(d['ms_per_step'], 3), 'policy', d['config']['policy'], 'frac', round(rf['frac'], 3),
      'kernel_ms', rf.get('kernel_ms') and round(rf['kernel_ms'], 3), 'step_frac', rf.get('step') and round(rf['step']['frac'], 3))
print('e2e', round(d['e2e']['value']), 'cpu', d.get('cpu_baseline') and round(d['cpu_baseline']['value'], 2), 'clocks', d['clocks'], 'cusparse', d.get('cusparse') and round(d['cusparse'].get('ms', 0), 3))
for p, r in d['policies'].items():
    lm = r.get('lru_model', {})
    print(f"{p:12s} {r['ms']:7.3f} ms {r['gflops']:7.0f} GF/s frac {r['roofline_frac']:.3f} ceil {lm.get('ceiling_frac', 0):.3f} build {r['build_ms']:8.1f} ms")

import json, sys
for f in sys.argv[1:]:
    print(f)
    for l in open(f):
        l = l.strip()
        if not l.startswith("{"):
            continue
        d = json.loads(l); r = d['roofline']
        print(f"  {d['config'].get('kernel','-'):8s} {str(d['config'].get('launch')):28s} value {d['value']:.4e} ms {d['ms_per_step']:.4f} "
              f"step {d.get('gbps',0):.0f} GB/s kern {r['achieved']:.0f} GB/s frac {r['frac']:.3f} share {r.get('share_of_step',0):.3f} "
              f"clk {d['clocks']['sm_mhz']} {d['clocks']['reasons']} copy {d.get('copy_gbs_same_box',0):.0f}")
        if d.get('e2e'): print('   e2e', round(d['e2e']['value']/1e9,2), 'G/s', round(d['e2e']['ms_per_step'],3), 'ms')
        if d.get('cpu_baseline'): print('   cpu', d['cpu_baseline']['value'])

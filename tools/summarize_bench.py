"""Print the key numbers of a bench JSON line."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(f"value {d['value']/1e6:.1f} M nodes/s  ms/step {d['ms_per_step']:.3f}  e2e {d['e2e']['value']/1e6:.1f} M nodes/s")
r = d["roofline"]
print(f"roofline[{r['kernel']}] {r['achieved']:.0f} GB/s = {100*r['frac']:.1f}% of {r['peak']}")
rl = d["relocate"]
print(f"relocate {rl['GB/s']:.0f} GB/s ({100*rl['frac_of_peak']:.1f}%) {rl['avg_us']:.1f} us")
su = d.get('sustained_relocate')
if su: print(f"sustained relocate x{su['replicas']}: {su['GB/s']:.0f} GB/s ({100*su['frac_of_peak']:.1f}%) {su['avg_ms']:.3f} ms/call {su['nodes_per_s']/1e9:.2f} G nodes/s")
ip = d.get('relocate_in_place')
if ip:
    for k, v in ip.items():
        if isinstance(v, dict): print(f"in place {k}: {v['avg_us']:.1f} us {v['GB/s']:.0f} GB/s ({100*v['frac_of_peak']:.1f}%) {v['nodes_per_s']/1e9:.2f} G nodes/s")
bu = d.get('buffers')
if bu: print(f"buffers: {bu['n_perm']} perm ({bu['blob_bytes']/1e6:.2f} MB) plan {bu['plan_ms']:.3f} ms save {bu['save_us']:.1f} us restore {bu['restore_us']:.1f} us = {bu['restore_GB/s']:.0f} GB/s ok={bu['restore_ok']} {bu['classes']}\n   kernels {bu.get('kernel_us')} events {bu.get('restore_events_GB/s', 0):.0f} GB/s")
for k, v in d["kernels"].items():
    print(f"  {k:22s} n={v['launches']:4d} avg {v['avg_us']:8.2f} us  share {100*v['share_of_step']:5.1f}%  " +
          (f"{v['GB/s']:.0f} GB/s" if 'GB/s' in v else ""))
print("cpu", d.get("cpu_baseline"), "clocks", d.get("clocks"), "launches", d.get("gpu_launches"))

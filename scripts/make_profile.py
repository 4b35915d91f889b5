"""profiles/<round>_eval32_<cfg>_ncu.json from an ncu --set full report (run here, not on the box).

usage: python scripts/make_profile.py REPORT.ncu-rep CONFIG COMMAND [LAUNCH_CSV] [TAG]
"""
import json, os, shutil, sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summary  # noqa: E402

rep, cfg, cmd = sys.argv[1], sys.argv[2], sys.argv[3]
s = summary(rep)[0]
keys = [k for k in s if not k.endswith('.unit') and k not in ('kernel', 'stall_cycles_per_issue')]
metrics = {k: {'value': s[k], 'unit': s.get(k + '.unit', '')} for k in keys}
scale = {'Tbyte': 1e12, 'Gbyte': 1e9, 'Mbyte': 1e6, 'Kbyte': 1e3, 'byte': 1.0}
dram = sum(s[k] * scale[s[k + '.unit']] for k in ('dram__bytes_read.sum', 'dram__bytes_write.sum'))
lts = None
if s.get('lts__t_bytes.sum') is not None:
    lts = s['lts__t_bytes.sum'] * scale.get(s['lts__t_bytes.sum.unit'], 1.0)
if lts is None and s.get('lts__t_sectors_srcunit_tex_op_read.sum') is not None:
    # L2 traffic from the SMs (L1 misses, stores and reductions): 32-byte sectors
    lts = 32.0 * (s['lts__t_sectors_srcunit_tex_op_read.sum'] +
                  s['lts__t_sectors_srcunit_tex_op_write.sum'])
dur = s['gpu__time_duration.sum'] * {'ms': 1e-3, 'us': 1e-6, 'ns': 1e-9}[s['gpu__time_duration.sum.unit']]
tag = sys.argv[5] if len(sys.argv) > 5 else 'r2'
out = {'kernel': s['kernel'], 'config': cfg, 'command': cmd, 'round': int(tag[1]), 'metrics': metrics,
       'stall_cycles_per_issue': s['stall_cycles_per_issue'],
       'dram_bytes_per_launch': dram, 'duration_s': dur, 'lts_bytes_per_launch': lts,
       'dram_GBps': dram / dur / 1e9,
       'l2_GBps': (lts / dur / 1e9) if lts else None,
       'note': 'one launch, ncu --set full --clock-control none (cold, serialised): compare '
               'shares and counters, not the absolute time, with bench.py'}
name = os.path.join('profiles', f"{tag}_eval32_{cfg}_ncu.json")
json.dump(out, open(name, 'w'), indent=1)
print('wrote', name, round(dram / 1e9, 3), 'GB', round(dur * 1e3, 3), 'ms')
if len(sys.argv) > 4:
    dst = os.path.join('profiles', f"{tag}_launches_{cfg}.csv")
    shutil.copy(sys.argv[4], dst)
    print('copied', dst)

"""Static check of JIT register forwarding on saved PTX (RTLSIM_JIT_SAVE=dir,
generated with RTLSIM_JIT_FWD=0): replays the forwarding rule of jit.cpp per
warp and step and reports every forwarded read across which ANOTHER warp wrote
a physically overlapping shared-memory range (any layout) — the condition the
rule must exclude. python tools/fwd_hazard_check.py <dir>"""
import re, sys, glob, collections
rx_st = re.compile(r'^\s*(@%\w+\s+)?st\.shared\.(u32|u16|u8)\s+\[%(rw|rh|rb|smb)\+(\d+)\]')
rx_ld = re.compile(r'^\s*(@%\w+\s+)?ld\.shared\.(u32|u16|u8)\s+%r\d+,\s+\[%(rw|rh|rb|smb)\+(\d+)\]')
rx_cp = re.compile(r'^\s*(@%(\w+)\s+)?cp\.async\.ca\.shared\.global\s+\[%(rw|smb)\+(\d+)\]')
def phys(space, off, pred=None):
    w = off // 4
    if space == 'smb': return (w, w + 1)
    if space == 'rw':
        n = 32 if pred is None else {'pl16': 16, 'pl8': 8, 'pl0': 1}[pred]
        return (w, w + n)
    if space == 'rh': return (w, w + 16)
    if space == 'rb': return (w, w + 8)
SP = {'rw': 'W', 'rh': 'H', 'rb': 'B', 'smb': 'S'}
def analyse(path, fwd_max=2):
    txt = open(path).read()
    bad = 0
    for fn in re.split(r'\n\.func ', txt)[1:]:
        # warp sections
        parts = re.split(r'\n(\$W\d+):\n', fn)
        if len(parts) == 1: secs = [('W0', parts[0])]
        else: secs = [(parts[i], parts[i + 1]) for i in range(1, len(parts), 2)]
        events = []   # (warp, step, kind, key, phys)
        for wi, (lab, body) in enumerate(secs):
            step = 0
            for line in body.split('\n'):
                if 'bar.sync' in line: step += 1; continue
                m = rx_st.match(line)
                if m:
                    sp, off = m.group(3), int(m.group(4))
                    events.append((wi, step, 'w', (SP[sp], off // 4), phys(sp, off))); continue
                m = rx_cp.match(line)
                if m:
                    pred, sp, off = m.group(2), m.group(3), int(m.group(4))
                    key = ('S', off // 4) if sp == 'smb' else ({'pl16': 'H', 'pl8': 'B'}.get(pred, 'W'), off // 4)
                    events.append((wi, step, 'c', key, phys(sp, off, pred))); continue
                m = rx_ld.match(line)
                if m and not m.group(1):
                    sp, off = m.group(3), int(m.group(4))
                    events.append((wi, step, 'r', (SP[sp], off // 4), phys(sp, off)))
        writes = collections.defaultdict(list)
        for (w, s, k, key, ph) in events:
            if k in 'wc': writes[key].append((s, w)); 
        allw = [(w, s, ph) for (w, s, k, key, ph) in events if k in 'wc']
        for wi in range(len(secs)):
            fwd = {}
            for (w, s, k, key, ph) in events:
                if w != wi: continue
                if k == 'w': fwd[key] = (s, ph); continue
                if k == 'c': fwd.pop(key, None); continue
                if key in fwd:
                    s0, ph0 = fwd[key]
                    impl_ok = s - s0 <= fwd_max and not any(ww != wi and s0 < ss <= s for (ss, ww) in writes[key])
                    if impl_ok:
                        true_ok = not any(ww != wi and s0 < ss <= s and p[0] < ph[1] and ph[0] < p[1] for (ww, ss, p) in allw)
                        if not true_ok:
                            bad += 1
                            if bad <= 5: print(path, 'warp', wi, 'key', key, 'fwd from step', s0, 'read at', s)
                    else:
                        fwd[key] = (s - 1, ph)
                else:
                    fwd[key] = (s - 1, ph)
    return bad
tot = 0
for p in sorted(glob.glob(sys.argv[1] + '/part*.ptx')):
    tot += analyse(p)
print('hazards', tot)

"""Summarise bench JSON lines: ms, c, parity, phases, prepared."""
import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        print(f, "ERR"); continue
    ph = (d.get("roofline") or {}).get("phase_ms_per_step", {})
    pr = d.get("prepared") or {}
    par = (d.get("parity") or {}).get("ok")
    s = f"{f:38s} {d['ms_per_step']:8.3f} c={d['config'].get('window_bits')} par={par} " + " ".join(f"{k[:4]}={v:.3f}" for k, v in ph.items())
    if pr:
        s += f" | prep {pr['ms_per_step']:.3f} c={pr.get('window_bits')} " + " ".join(f"{k[:4]}={v:.3f}" for k, v in pr.get('phase_ms_per_step', {}).items())
    print(s)

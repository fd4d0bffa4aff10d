"""Static single-warp cycle estimate of the loops in a cubin / object (development tool).

Reads `cuobjdump -sass` output, decodes each instruction's control bits (stall count, write /
read scoreboard slots, wait mask; B300_MICROARCH.md "Per-warp issue scheduler") and runs the
guide's single-warp issue model over every innermost backward-branch loop twice (the second
pass is reported, so loop-carried scoreboard waits are counted).  Variable-latency ops get the
latencies below (B200 measurements from tools/micro/lat.cu; L2 for global loads).

    python tools/sass_cycles.py build/ad_gen_lcs_r6e2w1.cu.o [--marker VIMNMX3] [--steps 16]
"""
import argparse
import re
import subprocess

VAR_LAT = {"SHFL": 27, "LDS": 29, "LDSM": 29, "LDG": 260, "LD": 260, "R2UR": 10, "S2R": 20, "S2UR": 20,
           "CS2R": 20, "LDC": 20, "LDCU": 20, "ATOMS": 30, "VOTEU": 10, "MATCH": 20, "REDUX": 20,
           "POPC": 10, "FLO": 10, "BREV": 10, "I2F": 10, "F2I": 10, "MUFU": 20}


def parse(path, kernel=None):
    txt = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True, check=True).stdout
    funcs = {}
    cur = None
    lines = txt.splitlines()
    i = 0
    while i < len(lines):
        l = lines[i]
        m = re.match(r"\s*Function : (\S+)", l)
        if m:
            cur = m.group(1)
            funcs[cur] = []
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?)\s*;?\s*/\* (0x[0-9a-f]{16}) \*/", l)
        if m and cur is not None and i + 1 < len(lines):
            m2 = re.match(r"\s*/\* (0x[0-9a-f]{16}) \*/", lines[i + 1])
            hi = int(m2.group(1), 16) if m2 else 0
            ctl = hi >> 41
            funcs[cur].append({
                "addr": int(m.group(1), 16), "text": m.group(2),
                "stall": ctl & 0xF, "yield": (ctl >> 4) & 1, "wbar": (ctl >> 5) & 7,
                "rbar": (ctl >> 8) & 7, "wait": (ctl >> 11) & 0x3F,
            })
            i += 2
            continue
        i += 1
    if kernel:
        funcs = {k: v for k, v in funcs.items() if kernel in k}
    return funcs


def opname(text):
    t = re.sub(r"^@!?U?P[T0-9]+\s+", "", text)
    return t.split()[0] if t else ""


def simulate(body, passes=2):
    sb = [0.0] * 6
    T = 0.0
    start = 0.0
    for p in range(passes):
        if p == passes - 1:
            start = T
        for ins in body:
            arm = max([sb[s] for s in range(6) if ins["wait"] >> s & 1] or [0.0])
            T = max(T, arm)
            op = opname(ins["text"]).split(".")[0]
            lat = VAR_LAT.get(op, 20)
            if ins["wbar"] < 6:
                sb[ins["wbar"]] = max(sb[ins["wbar"]], T + lat)
            if ins["rbar"] < 6:
                sb[ins["rbar"]] = max(sb[ins["rbar"]], T + 6)
            T += max(ins["stall"], 1)
    return T - start


def loops(ins):
    addr2i = {x["addr"]: k for k, x in enumerate(ins)}
    out = []
    for k, x in enumerate(ins):
        m = re.search(r"BRA(\.U)?\s.*?(0x[0-9a-f]+)", x["text"])
        if m:
            tg = int(m.group(2), 16)
            if tg < x["addr"] and tg in addr2i:
                out.append((addr2i[tg], k))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("obj")
    ap.add_argument("--kernel", default=None)
    ap.add_argument("--marker", default="VIMNMX3")
    ap.add_argument("--steps", type=int, default=0, help="steps per loop iteration (prints cycles/step)")
    ap.add_argument("--dump", action="store_true")
    ap.add_argument("--all", action="store_true", help="also loops that contain inner loops (e.g. spin waits)")
    ap.add_argument("--count", type=int, default=0, help="only loops with exactly this many marker instructions")
    a = ap.parse_args()
    for fn, ins in parse(a.obj, a.kernel).items():
        for j, k in loops(ins):
            body = ins[j:k + 1]
            # innermost loops only: no other backward branch inside
            if not a.all and any(j < jj and kk < k for jj, kk in loops(ins)):
                continue
            nm = sum(a.marker in b["text"] for b in body)
            if nm == 0 or (a.count and nm != a.count):
                continue
            cyc = simulate(body)
            stalls = sum(max(b["stall"], 1) for b in body)
            ops = {}
            for b in body:
                o = opname(b["text"])
                ops[o] = ops.get(o, 0) + 1
            top = ", ".join(f"{o} {c}" for o, c in sorted(ops.items(), key=lambda x: -x[1])[:8])
            ps = f"  {cyc / a.steps:.1f} cyc/step" if a.steps else ""
            print(f"{fn[:60]} loop {body[0]['addr']:#x}-{body[-1]['addr']:#x}: {len(body)} instr, "
                  f"{a.marker} {nm}, stall-sum {stalls}, sim {cyc:.0f} cyc{ps}\n    {top}")
            if a.dump:
                for b in body:
                    print(f"    {b['addr']:05x} s{b['stall']:2d} w{b['wbar']} r{b['rbar']} m{b['wait']:02x}  {b['text']}")


if __name__ == "__main__":
    main()

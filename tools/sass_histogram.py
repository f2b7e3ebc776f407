"""SASS instruction histogram of lib/libft2.so (cuobjdump -sass): the
mnemonics that prove tcgen05 / TMEM / TMA / DSMEM use, totals and per kernel.
python tools/sass_histogram.py > profiles/r2_sass_histogram.txt"""
import collections, os, re, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "lib", "libft2.so")
KEYS = ["UTCHMMA", "UTCHMMA.2CTA", "UTCBAR", "UTCBAR.2CTA", "UTMALDG", "UTMAPF", "UTMACCTL", "UBLKPF", "LDTM",
        "STAS", "SYNCS", "UCGABAR_ARV", "UCGABAR_WAIT", "VIMNMX", "CREDUX", "REDUX", "ATOMG", "LDG", "STG", "LDL", "STL"]
sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
per, cur = collections.OrderedDict(), None
for line in sass.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        cur = m.group(1)
        per[cur] = collections.Counter()
        continue
    m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*(?:\.2CTA)?)", line)
    if cur and m:
        op = m.group(1)
        base = op.split(".")[0]
        for k in KEYS:
            if op == k or (k == base and "." not in k):
                per[cur][k] += 1
tot = collections.Counter()
for c in per.values():
    tot.update(c)
print("# SASS instruction histogram of lib/libft2.so (cuobjdump -sass, sm_100a), round 2 session e")
print("# tcgen05 MMA = UTCHMMA (.2CTA = cta_group::2), commit = UTCBAR, TMA = UTMALDG/UTMAPF,")
print("# TMEM load = LDTM, DSMEM st.async = STAS, mbarrier = SYNCS, cluster barrier = UCGABAR_*, local memory = LDL/STL")
print("\n## totals")
for k in KEYS:
    print(f"{k:14s} {tot[k]}")
print("\n## per kernel (kernels using tcgen05 / TMA / key-space min-max / local memory)")
for name, c in per.items():
    if any(c[k] for k in ("UTCHMMA", "UTMALDG", "VIMNMX", "LDL", "STL", "LDTM")):
        print(name[:110])
        print("    " + ", ".join(f"{k} {c[k]}" for k in KEYS if c[k]))

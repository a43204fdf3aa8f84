"""Write the SASS of the production rhs kernel(s) to profiles/ with opcode
counts that prove the TMA / mbarrier / FP64 mix (cuobjdump -sass of the
in-tree library; encodings stripped).  usage: python tools/sass_listing.py OUT"""
import re
import subprocess
import sys
from collections import Counter

sys.path.insert(0, ".")
from paper_conf_icpp_tiankexc16_b200 import _abi  # noqa: E402

out = sys.argv[1]
names = ["_ZN6safara21rhs_kernel_fast_ws_udE14CUtensorMap_stS0_NS_6ParamsE",
         "_ZN6safara18rhs_kernel_fast_udE14CUtensorMap_stS0_NS_6ParamsE"]
with open(out, "w") as fh:
    for fn in names:
        sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", "-fun", fn, _abi.LIB_PATH],
                              capture_output=True, text=True).stdout
        ins = []
        for line in sass.splitlines():
            m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
            if m:
                ins.append((m.group(1), m.group(2).strip()))
        ops = Counter(re.sub(r"^@!?U?P\w+\s+", "", t).split()[0] for _, t in ins)
        fam = Counter()
        for op, c in ops.items():
            fam[op.split(".")[0]] += c
        fh.write(f"== {fn}\n")
        fh.write(f"instructions: {len(ins)}\n")
        keys = ["UTMALDG", "UTMASTG", "UBLKCP", "SYNCS", "USETMAXREG", "DFMA", "DMUL", "DADD",
                "MUFU", "LDS", "STS", "LDG", "STG", "SHFL", "STL", "LDL"]
        fh.write("counts: " + ", ".join(f"{k}={fam.get(k, 0)}" for k in keys) + "\n")
        for a, t in ins:
            fh.write(f"/*{a}*/ {t}\n")
        fh.write("\n")
print(open(out).read().split("\n== ")[0][:600])

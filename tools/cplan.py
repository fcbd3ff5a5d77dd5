"""Emit a plan-specialised kernel header (kernel.cu STM_CPLAN build): the compiled device plan of
one query as a constant record.  usage: python tools/cplan.py PATTERN OUT.h [vi] [labels=0,1,..]
Build with: python paper_conf_sc_weij22_b200/build.py --out=variants/libstm_X.so STM_CPLAN=1 \\
            'STM_CPLAN_HEADER="/abs/OUT.h"'   (the launch must use the same plan)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen  # noqa: E402
from paper_conf_sc_weij22_b200 import stm  # noqa: E402

name, out = sys.argv[1], sys.argv[2]
vi = "vi" in sys.argv[3:]
lab = None
for a in sys.argv[3:]:
    if a.startswith("labels="):
        lab = tuple(int(x) for x in a[7:].split(","))
p = stmgen.CATALOG[name]
plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi)
raw = stm.stm_plan_raw(plan.handle)
with open(out, "w") as f:
    f.write(f"// plan-specialised kernel: {name} vi={vi} labels={lab}\n// {plan.describe().splitlines()[0]}\n")
    f.write(f"#define STM_CPLAN_K {p.k}\n")
    f.write("__device__ const StmPlanBytes kCPlan = {{" + ",".join(str(b) for b in raw) + "}};\n")
print(out, len(raw), "bytes")

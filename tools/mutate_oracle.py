"""Mutation test of the oracle's pins: apply each source mutation to a scratch copy of the
repo's oracle/hmg_oracle.c, run the CPU pins (tests/test_oracle.py), and report whether some
pin fails (killed) or all pass (survived).
usage: python tools/mutate_oracle.py > profiles/oracle_mutants_<tag>.txt"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MUTANTS = [
    ("vit_pass uses msv_nats", "return !(or_pvalue(or_vit_nats(raw, L)", "return !(or_pvalue(or_msv_nats(raw, L)"),
    ("MSV J->B re-entry dropped", "xB = sat_u8((xJ > base ? xJ : base) - tjb);", "xB = sat_u8(base - tjb);"),
    ("MSV tec dropped", "int e = sat_u8(xE - tec);", "int e = sat_u8(xE);"),
    ("MSV overflow > for >=", "if (xE >= 255 - bias) return 255;", "if (xE > 255 - bias) return 255;"),
    ("MSV diagonal k for k-1", "int s = prev[k - 1] > xBp ? prev[k - 1] : xBp;", "int s = prev[k] > xBp ? prev[k] : xBp;"),
    ("MSV tbm dropped", "int xBp = sat_u8(xB - tbm);", "int xBp = sat_u8(xB);"),
    ("MSV bias dropped", "s = sat_u8(s + bias);", "s = sat_u8(s);"),
    ("VF tMD index", "sat_s16(Mn[k - 1] + tMD[k - 2])", "sat_s16(Mn[k - 1] + tMD[k - 1])"),
    ("VF tDD index", "int dd = sat_s16(Dn[k - 1] + tDD[k - 2]);", "int dd = sat_s16(Dn[k - 1] + tDD[k - 1]);"),
    ("VF tIM index", "int im = sat_s16(Ip[k - 1] + tIM[k - 1]);", "int im = sat_s16(Ip[k - 1] + tIM[k - 2 < 0 ? 0 : k - 2]);"),
    ("VF DM from I", "int dm = sat_s16(Dp[k - 1] + tDM[k - 1]);", "int dm = sat_s16(Ip[k - 1] + tDM[k - 1]);"),
    ("VF D->D closure dropped", "if (dd > Dn[k]) Dn[k] = dd;", "(void)dd;"),
    ("VF overflow > for >=", "if (xE >= 32767) return 32767;", "if (xE > 32767) return 32767;"),
    ("VF xJ not fed back", "xB = (xJ > xN ? xJ : xN) + move;", "xB = xN + move;"),
    ("VF E->C dropped", "int e = xE + xE_w;", "int e = xE;"),
    ("VF I self-loop dropped", "int ii = sat_s16(Ip[k] + tII[k - 1]);", "int ii = -32768;"),
    ("VF emission dropped", "Mn[k] = sat_s16(m + rsc[x * M + (k - 1)]);", "Mn[k] = sat_s16(m);"),
    ("null1 p1 sign", "return (float)((float)L * log((double)p1) + log(1.0 - (double)p1));",
     "return (float)((float)L * log((double)p1) - log(1.0 - (double)p1));"),
    ("Gumbel sign", "double y = lambda * (x - mu);", "double y = lambda * (mu - x);"),
    ("pass >= for >", "return !(or_pvalue(or_msv_nats(raw, L), L, mu, lambda) > F);",
     "return !(or_pvalue(or_msv_nats(raw, L), L, mu, lambda) >= F);"),
    ("roundf -> truncation", "float c = -1.0f * roundf(or_scale_b() * s);\n  if (c > 255.0f)",
     "float c = -1.0f * truncf(or_scale_b() * s);\n  if (c > 255.0f)"),
    ("II clamp dropped", "if (t == 6 && v > -1) v = -1;", ""),
    ("vit nats -3 dropped", "sc /= or_scale_w();\n  sc -= 3.0;", "sc /= or_scale_w();"),
    ("Forward D->E dropped", "E = or_lse(E, or_lse(Mn[k], Dn[k]));", "E = or_lse(E, Mn[k]);"),
]


def main():
    src = open(os.path.join(ROOT, "oracle", "hmg_oracle.c")).read()
    tmp = tempfile.mkdtemp(prefix="mut_")
    for d in ("oracle", "tests", "paper_conf_ipps_jiangg15_b200"):
        shutil.copytree(os.path.join(ROOT, d), os.path.join(tmp, d),
                        ignore=shutil.ignore_patterns("*.so", "_build", "__pycache__", "csrc"))
    shutil.copy(os.path.join(ROOT, "pytest.ini"), tmp)
    killed = 0
    for name, a, b in MUTANTS:
        if a not in src:
            print("| %s | pattern not found |" % name)
            continue
        open(os.path.join(tmp, "oracle", "hmg_oracle.c"), "w").write(src.replace(a, b, 1))
        for f in os.listdir(os.path.join(tmp, "oracle")):
            if f.endswith(".so"):
                os.remove(os.path.join(tmp, "oracle", f))
        r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-m", "not gpu", "-n", "8",
                            "tests/test_oracle.py"], cwd=tmp, capture_output=True, text=True)
        ok = r.returncode != 0
        killed += ok
        last = [l for l in r.stdout.splitlines() if l.startswith("FAILED")][:1]
        print("| %s | %s | %s |" % (name, "killed" if ok else "SURVIVED", last[0][7:90] if last else ""), flush=True)
    print("\n%d / %d mutants killed" % (killed, len(MUTANTS)))
    shutil.rmtree(tmp)


if __name__ == "__main__":
    main()

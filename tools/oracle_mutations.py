"""Mutation check of the oracle pins: inject one plausible misreading at a time
into a COPY of oracle/capgpu_oracle.c, build it to a scratch library, run the
named pin tests against it (CAPGPU_ORACLE_LIB points oracle.py at the scratch
library), and report whether the pins caught it.  The committed oracle is
never modified.  usage: python tools/oracle_mutations.py [> profiles/....txt]"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "capgpu_oracle.c")

# (name, old, new, tests)
MUTATIONS = [
    ("S4: gamma applied to the CPU capacity",
     "g[l] = (j == 0) ? lv / c->f_max[j] : pow(lv / c->f_max[j], c->gamma);",
     "g[l] = pow(lv / c->f_max[j], c->gamma);", "tests/test_oracle_thr_budget.py"),
    ("S4: capacity f_max/level inverted",
     "g[l] = (j == 0) ? lv / c->f_max[j] : pow(lv / c->f_max[j], c->gamma);",
     "g[l] = (j == 0) ? lv / c->f_max[j] : pow(c->f_max[j] / lv, c->gamma);", "tests/test_oracle_thr_budget.py"),
    ("S4: missing 1/S on the throughput", "    thr[j] = tsum * inv_s;", "    thr[j] = tsum;",
     "tests/test_oracle_thr_budget.py"),
    ("S4: thr_max dropped from the capacity", "tsum = tsum + dmin(dem[j], thr_max[j] * g[l]);",
     "tsum = tsum + dmin(dem[j], g[l]);", "tests/test_oracle_thr_budget.py"),
    ("S5: caps from the weights of instant k (no lag)",
     "    for (int i = 0; i < n_servers; ++i) wprev_v[i] = sv[i].w_prev;\n    ora_budget_caps(",
     "    for (int i = 0; i < n_servers; ++i) wprev_v[i] = mean_theta(c, sv[i].thr, sv[i].thr_max);\n"
     "    ora_budget_caps(", "tests/test_oracle_thr_budget.py"),
    ("S5: rack limit dropped", "double Br = dmin(B_rack_max[r], Pr + (B_c - pmin_tot) * Wr / W);",
     "double Br = Pr + (B_c - pmin_tot) * Wr / W;", "tests/test_oracle_thr_budget.py"),
    ("S5: cap not proportional to w_i", "cap[i] = pmin[i] + (Br - Pr) * w[i] / Wr;",
     "cap[i] = pmin[i] + (Br - Pr) / (double)rack;", "tests/test_oracle_thr_budget.py"),
]


def main():
    src = open(SRC).read()
    tmp = tempfile.mkdtemp()
    ok = True
    for name, old, new, tests in MUTATIONS:
        assert src.count(old) == 1, f"mutation anchor not unique/found: {name}"
        odir = os.path.join(tmp, "oracle")
        os.makedirs(odir, exist_ok=True)
        if not os.path.exists(os.path.join(tmp, "gen")):
            os.symlink(os.path.join(ROOT, "gen"), os.path.join(tmp, "gen"))
        msrc = os.path.join(odir, "capgpu_oracle.c")
        open(msrc, "w").write(src.replace(old, new))
        shutil.copy(os.path.join(ROOT, "oracle", "capgpu_oracle.h"), odir)
        lib = os.path.join(odir, "libmut.so")
        subprocess.run(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-std=c11", "-shared", "-fPIC",
                        "-o", lib, msrc, "-lm"], check=True, capture_output=True)
        env = dict(os.environ, CAPGPU_ORACLE_LIB=lib)
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "not gpu", tests], cwd=ROOT,
                           env=env, capture_output=True, text=True)
        caught = r.returncode != 0
        ok &= caught
        last = [ln for ln in r.stdout.splitlines() if ln.strip()][-1] if r.stdout.strip() else ""
        print(f"{'CAUGHT ' if caught else 'MISSED '} {name:55s} | {last}")
    shutil.rmtree(tmp, ignore_errors=True)
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()

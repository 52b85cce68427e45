"""Mutation check of the oracle's pins (VERDICT r01 "What's weak" 1): every mutant below is a plausible
mistake in one branch of oracle/snn_oracle.c; each must turn at least one `-m "not gpu"` test red.

Runs in a scratch copy of the repository (the tree itself is never modified):
    python tools/oracle_mutants.py            # all mutants
    python tools/oracle_mutants.py M1 M2      # a subset
Prints one line per mutant: KILLED (some test failed) or SURVIVED, and exits 1 if any survived."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, passage, original line fragment, mutated fragment)
MUTANTS = [
    ("M1", "P:88 t_inh, R7 HOLD keeps v",
     "if (p->inh_mode == 0) { n->v_f[j] = n->vresetf; n->v_x[j] = n->Vreset; }",
     "{ n->v_f[j] = n->vresetf; n->v_x[j] = n->Vreset; }"),
    ("M2", "P:84 eqs.(4)(5), R16 window t - last_pre <= t_LTP",
     "(t - n->last_pre[i]) <= p->t_ltp_steps", "(t - n->last_pre[i]) < p->t_ltp_steps"),
    ("M3", "P:85 eq.(7), R10 Dt = t - last_post",
     "int D = t - n->last_post[j];", "int D = t - n->last_post[j] + 1;"),
    ("M4", "P:85 eq.(6), R14 LTP sees this step's pre spikes (D = 0)",
     "int D = t - n->last_pre[i];\n          if (D >= n->L_pot) continue;",
     "int D = t - n->last_pre[i];\n          if (D == 0 || D >= n->L_pot) continue;"),
    ("M5", "R7 ties -> lowest index",
     "(n->v_x[j] > n->v_x[W]) : (n->v_f[j] > n->v_f[W])", "(n->v_x[j] >= n->v_x[W]) : (n->v_f[j] >= n->v_f[W])"),
    ("M6", "P:89 clamp at q_max",
     "if (*qq < n->q_max) *qq += 1;", "*qq += 1;"),
    ("M7", "R6 refractory: held neurons do not integrate",
     "if (n->cnt[j] > 0) { n->cnt[j]--; cand[j] = 0; continue; }",
     "if (n->cnt[j] > 0) { n->cnt[j]--; cand[j] = 0; }"),
    ("M8", "R7 lone LAYER spiker not self-inhibited",
     "int other = (nsp >= 2) || (j != spikers[0]);", "int other = 1;"),
    # 32-bit floating-point conductance arm (NEXT-2, R28)
    ("M9", "P:84 eq.(4) normalised by (G_max - G_min)",
     "return p->alpha_p * oracle_exp_recipe(n, -p->beta_p * ((double)G - p->g_min) / span);",
     "return p->alpha_p * oracle_exp_recipe(n, -p->beta_p * ((double)G - p->g_min));"),
    ("M10", "P:84 eq.(5) uses alpha_d / beta_d",
     "return p->alpha_d * oracle_exp_recipe(n, -p->beta_d * (p->g_max - (double)G) / span);",
     "return p->alpha_d * oracle_exp_recipe(n, -p->beta_p * (p->g_max - (double)G) / span);"),
    ("M11", "P:83 eq.(3) I = v_pre sum g (32 bit)",
     "float I  = Sg * n->kV;", "float I  = Sg * n->kI;"),
    ("M12", "P:89 LTD of the 32-bit arm subtracts eq.(5)",
     "*g = g_step(n, *g, oracle_dg(n, 1, *g), 1);", "*g = g_step(n, *g, oracle_dg(n, 0, *g), 1);"),
    ("M13", "R28 exp recipe: Cody-Waite low part",
     "r = fma(-k, LN2_LO, r);", "r = fma(k, LN2_LO, r);"),
    ("M14", "R28 clamp at G_max",
     "if (G1 > n->gmaxf) G1 = n->gmaxf;", ""),
    ("M15", "R16 window at 32 bits (fp32 branch sees pot)",
     "double dG = oracle_dg(n, !pot, *g);", "double dG = oracle_dg(n, pot, *g);"),
]


def run(names):
    survived = []
    for name, passage, orig, mut in MUTANTS:
        if names and name not in names:
            continue
        with tempfile.TemporaryDirectory() as tmp:
            dst = os.path.join(tmp, "repo")
            shutil.copytree(ROOT, dst, ignore=shutil.ignore_patterns(".git", "gpurun_out", "profiles", "*.so"))
            src = os.path.join(dst, "oracle", "snn_oracle.c")
            text = open(src).read()
            assert text.count(orig) == 1, f"{name}: fragment not found exactly once"
            open(src, "w").write(text.replace(orig, mut))
            subprocess.run(["gcc", "-std=c11", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-o",
                            os.path.join(dst, "oracle", "liboracle.so"), src, "-lm"], check=True)
            r = subprocess.run([sys.executable, "-m", "pytest", "tests", "-x", "-q", "-m", "not gpu",
                                "-p", "no:cacheprovider", "--deselect", "tests/test_abi.py"],
                               cwd=dst, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
            tail = [l for l in r.stdout.splitlines() if l.startswith("FAILED")][:1]
            verdict = "KILLED" if r.returncode != 0 else "SURVIVED"
            if r.returncode == 0:
                survived.append(name)
            print(f"{name:3s} {verdict:8s} {passage:55s} {tail[0] if tail else ''}", flush=True)
    return survived


if __name__ == "__main__":
    sys.exit(1 if run(set(sys.argv[1:])) else 0)

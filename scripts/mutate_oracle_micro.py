"""Mutation check of the microphysics oracle's pins (tests/test_oracle_micro.py).

Each mutation is a plausible mistake in oracle/oracle.c's oracle_micro (a wrong constant,
exponent, sign, index or a dropped factor).  For each one the oracle, the input generator
and the pin file are copied to a scratch dir, the mutation applied to the copy of
oracle.c, and the pins run there; a mutation that passes every pin is a hole in the pins.
The unmutated copy must pass.  Run: python scripts/mutate_oracle_micro.py [-o out.txt]
"""
import argparse
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, old text in oracle.c, new text)
MUTATIONS = [
    ("evap: r01 survey diffusion term 2.55e8/(pc qvs)",
     "(2.55e6f * pc[k]) / (3.8f * qvs)", "2.55e8f / (pc[k] * qvs)"),
    ("evap: exponents 0.2046 <-> 0.525 swapped",
     "124.9f * oracle_pow_s(rq, 0.2046f)) *\n                                       oracle_pow_s(rq, 0.525f)",
     "124.9f * oracle_pow_s(rq, 0.525f)) *\n                                       oracle_pow_s(rq, 0.2046f)"),
    ("evap: ventilation constant 124.9 -> 12.49", "124.9f", "12.49f"),
    ("evap: ventilation offset 1.6 -> 0.16", "(1.6f + 124.9f", "(0.16f + 124.9f"),
    ("evap: conduction term 5.4e5 -> 5.4e4", "5.4e5f", "5.4e4f"),
    ("evap: diffusion constant 2.55e6 -> 2.55e5", "2.55e6f * pc[k]", "2.55e5f * pc[k]"),
    ("evap: density dropped from the rate", "/\n                                     (r[k] * qvs);",
     "/\n                                     (qvs);"),
    ("evap: deficit sign flipped", "max_s(qvs - QV[k], 0.0f)", "max_s(QV[k] - qvs, 0.0f)"),
    ("evap: no cap at the rain present", "fmin3(e1, max_s(-prod - QC[k], 0.0f), QR[k])",
     "min_s(e1, max_s(-prod - QC[k], 0.0f))"),
    ("evap: no cap at the saturation deficit", "fmin3(e1, max_s(-prod - QC[k], 0.0f), QR[k])",
     "min_s(e1, QR[k])"),
    ("evap: rate not multiplied by dt0", "((dt0 * (vent / dif))", "(((vent / dif))"),
    ("fall speed: density factor inverted", "sqrtf(RHO[0] / RHO[k])", "sqrtf(RHO[k] / RHO[0])"),
    ("fall speed: density factor dropped", "rhalf[k] = sqrtf(RHO[0] / RHO[k]);", "rhalf[k] = 1.0f;"),
    ("fall speed: constant 36.34 -> 3.634 (both sites)", "36.34f", "3.634f"),
    ("fall speed: exponent 0.1364 -> 0.2046 (both sites)", "0.1364f", "0.2046f"),
    ("sedimentation: receiving level's density -> source level's",
     "/ (r[k] * dz);", "/ (r[k + 1] * dz);"),
    ("sedimentation: top level a full cell", "(0.5f * dz)", "(dz)"),
    ("sedimentation: flux difference reversed", "(F[k + 1] - F[k])", "(F[k] - F[k + 1])"),
    ("substeps: dt0 = dt", "const float dt0 = dt / (float)nsub;", "const float dt0 = dt;"),
    ("substeps: precip not averaged", "precip[col] = prec / (float)nsub;", "precip[col] = prec;"),
    ("theta tendency: Exner factor dropped", "(2.5e6f / (1003.0f * PK[k]))", "(2.5e6f / (1003.0f))"),
    ("theta tendency: latent-heating sign flipped", "TH[k] = TH[k] + (2.5e6f", "TH[k] = TH[k] - (2.5e6f"),
    ("autoconversion: threshold 1e-3 -> 5e-4", "(QC[k] - 0.001f)", "(QC[k] - 0.0005f)"),
    ("accretion: constant 2.2 -> 0.22", "(dt0 * 2.2f)", "(dt0 * 0.22f)"),
    ("accretion: exponent 0.875 -> 0.525", "oracle_pow_s(QR[k], 0.875f)", "oracle_pow_s(QR[k], 0.525f)"),
    ("saturation: Tetens 17.27 -> 17.67", "(17.27f * (T - 273.0f))", "(17.67f * (T - 273.0f))"),
    ("saturation: F5 (Lv/cp dqvs/dT) halved", "const float F5 = 10214784.0f;",
     "const float F5 = 5107392.0f;"),
]


def run(tmp, mutation):
    src = os.path.join(ROOT, "oracle", "oracle.c")
    text = open(src).read()
    if mutation is not None:
        _, old, new = mutation
        assert old in text, f"mutation anchor not found: {old!r}"
        text = text.replace(old, new)
    work = tempfile.mkdtemp(dir=tmp)
    shutil.copytree(os.path.join(ROOT, "oracle"), os.path.join(work, "oracle"),
                    ignore=shutil.ignore_patterns("*.so", "__pycache__"))
    shutil.copytree(os.path.join(ROOT, "synthetic"), os.path.join(work, "synthetic"),
                    ignore=shutil.ignore_patterns("__pycache__"))
    os.makedirs(os.path.join(work, "tests"))
    for f in ("conftest.py", "test_oracle_micro.py"):
        shutil.copy(os.path.join(ROOT, "tests", f), os.path.join(work, "tests", f))
    open(os.path.join(work, "oracle", "oracle.c"), "w").write(text)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider",
                        "tests/test_oracle_micro.py"], cwd=work, capture_output=True, text=True)
    failed = [ln.split("::")[1].split(" ")[0] for ln in r.stdout.splitlines()
              if ln.startswith("FAILED")]
    return r.returncode, failed


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("-o", default=None)
    a = ap.parse_args()
    lines = []
    with tempfile.TemporaryDirectory() as tmp:
        rc, failed = run(tmp, None)
        lines.append(f"unmutated: rc={rc} failed={failed}")
        assert rc == 0, "the unmutated oracle must pass its pins"
        holes = 0
        for m in MUTATIONS:
            rc, failed = run(tmp, m)
            caught = rc != 0 and failed
            holes += not caught
            lines.append(f"{'CAUGHT' if caught else 'MISSED'}  {m[0]}: {len(failed)} pins fail "
                         f"({', '.join(sorted(set(f.split('[')[0] for f in failed)))})")
            print(lines[-1], flush=True)
        lines.append(f"{len(MUTATIONS) - holes}/{len(MUTATIONS)} mutations caught")
    print(lines[-1])
    if a.o:
        open(a.o, "w").write("\n".join(lines) + "\n")
    return 1 if holes else 0


if __name__ == "__main__":
    sys.exit(main())

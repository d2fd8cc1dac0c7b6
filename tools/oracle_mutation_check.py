"""Mutation check of the oracle pins: inject plausible definition mistakes into oracle/ one at a
time, run tests/test_oracle_closed_forms.py, report CAUGHT/MISSED, restore the file.
    python tools/oracle_mutation_check.py
"""
import subprocess, shutil, sys
muts = [
 ("oracle/transformer.py", "scale = 1.0 / np.sqrt(qh.shape[-1])", "scale = 1.0 / np.sqrt(qh.shape[-1] * qh.shape[1])", "1/sqrt(d) scale"),
 ("oracle/transformer.py", "q, k, v = qkv[..., :d], qkv[..., d:2 * d], qkv[..., 2 * d:]", "v, k, q = qkv[..., :d], qkv[..., d:2 * d], qkv[..., 2 * d:]", "q/v swapped"),
 ("oracle/transformer.py", "return t.reshape(B, S, h, d // h).transpose(0, 2, 1, 3)", "return t.reshape(B, S, d // h, h).transpose(0, 3, 1, 2)", "interleaved heads"),
 ("oracle/transformer.py", "    a, c1 = ln_fwd(x, p[\"ln1_g\"], p[\"ln1_b\"])", "    a, c1 = x, ln_fwd(x, p[\"ln1_g\"], p[\"ln1_b\"])[1]", "no pre-LN"),
 ("oracle/spos.py", "xp, xm = x[..., 0::2], x[..., 1::2]", "xp, xm = x[..., 1::2], x[..., 0::2]", "split parity"),
 ("oracle/spos.py", "return np.concatenate([xp, main], axis=-1), tapes", "return np.concatenate([main, xp], axis=-1), tapes", "concat order"),
 ("oracle/spos.py", "relu = kind == \"pw\" and (which == \"p\" or i == len(cl) - 1 or name in (\"m_pw1\", \"x_pw1\", \"x_pw2\"))", "relu = (kind == \"pw\" and (which == \"p\" or i == len(cl) - 1 or name in (\"x_pw1\", \"x_pw2\"))) or name == \"m_dw\"", "ReLU moved pw1->dw"),
 ("oracle/spos.py", "loss = float(np.mean(lse - logits[np.arange(B), labels]))", "loss = float(np.mean(lse - logits[np.arange(B), labels])) * 1.01", "CE scale"),
]
for f, a, b, what in muts:
    src = open(f).read()
    assert a in src, (f, a)
    open(f, "w").write(src.replace(a, b))
    try:
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "tests/test_oracle_closed_forms.py"], capture_output=True, text=True)
        last = r.stdout.strip().splitlines()[-1]
        print(f"{what:22s} -> {'CAUGHT' if r.returncode else 'MISSED'}: {last}")
    finally:
        open(f, "w").write(src)

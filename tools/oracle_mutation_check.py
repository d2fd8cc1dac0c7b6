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
 # the dense Conv 3x3 candidate (reading A40), caught by tests/test_oracle_spos.py's pins
 ("oracle/spos.py", "y += xp[:, u:u + s * (Ho - 1) + 1:s, v:v + s * (Wo - 1) + 1:s, :] @ w[:, u, v, :].T", "y += xp[:, u:u + s * (Ho - 1) + 1:s, v:v + s * (Wo - 1) + 1:s, :] @ w[:, v, u, :].T", "dense taps transposed", "tests/test_oracle_spos.py"),
 ("oracle/spos.py", "            dxp[sl] += dy @ w[:, u, v, :]", "            dxp[sl] += dy @ w[:, k - 1 - u, k - 1 - v, :]", "dense dgrad flipped", "tests/test_oracle_spos.py"),
 ("oracle/spos.py", "        L += [(\"m_pw1\", \"pw\", inp, mid, 1, 1), (\"m_cv\", \"cv\", mid, mid, k, s), (\"m_pw2\", \"pw\", mid, out, 1, 1)]", "        L += [(\"m_pw1\", \"pw\", inp, mid, 1, 1), (\"m_cv\", \"cv\", mid, mid, k, 1), (\"m_pw2\", \"pw\", mid, out, 1, 1)]", "dense stride ignored", "tests/test_oracle_spos.py"),
]
for m in muts:
    f, a, b, what = m[:4]
    test = m[4] if len(m) > 4 else "tests/test_oracle_closed_forms.py"
    src = open(f).read()
    assert a in src, (f, a)
    open(f, "w").write(src.replace(a, b))
    try:
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", test], capture_output=True, text=True)
        last = r.stdout.strip().splitlines()[-1]
        print(f"{what:22s} -> {'CAUGHT' if r.returncode else 'MISSED'}: {last}")
    finally:
        open(f, "w").write(src)

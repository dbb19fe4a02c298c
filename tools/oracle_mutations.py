"""Mutation check of the oracle pins: applies plausible mistakes to oracle/pf_oracle.c one at a time
and reports which pin catches each (restores the source afterwards). Run: python tools/oracle_mutations.py"""
import subprocess, shutil, sys
src='/root/repo/oracle/pf_oracle.c'
orig=open(src).read()
muts=[
 ("16.0 / (PI_D * PI_D)","8.0 / (PI_D * PI_D)"),
 ("(PI_D * p->eps / 4.0)","(PI_D * p->eps / 2.0)"),
 ("(4.0 * p->dx);\n    }","(2.0 * p->dx);\n    }"),
 ("xs[a] = ph[a] + f * (-r[a] + lam);","xs[a] = ph[a] + f * (r[a] - lam);"),
 ("return 6.0 * x * (1.0 - x);","return 3.0 * x * (1.0 - x);"),
 ("Q[i] += h * cT[i] * dTdt;","Q[i] += h * cT[i];"),
 ("Mf[i][j] += g_of(pb[a]) * s;","Mf[i][j] += h_of(pb[a]) * s;"),
 ("s += p->D[a][i][k] * chi[k][j];","s += chi[i][k] * p->D[a][k][j];"),
 ("(gr[a][d] / nrm_a);","(gr[L][d] / nrm_l);"),
 ("S[i] += c[i] * dh * dtphi;","S[i] -= c[i] * dh * dtphi;"),
 ("(chi[1][1] * rhs[0] - chi[0][1] * rhs[1]) / det","(chi[1][1] * rhs[0] - chi[1][0] * rhs[1]) / det"),
 ("s += p->gamma[a][b] * pb[b] * (pb[b] * dd[a] - pb[a] * dd[b]);","s += p->gamma[a][b] * pb[a] * (pb[b] * dd[a] - pb[a] * dd[b]);"),
 ("(double)z + (d == 2 ? 0.5 : 0.0)","(double)z"),
 ("double lam = rs / (double)N;","double lam = rs / (double)(N-1);"),
 ("om += gamma3_of(p, a, b, d) * ph[b] * ph[d];","om += 0.5*gamma3_of(p, a, b, d) * ph[b] * ph[d];"),
 ("r[a] = p->eps * (dadphi - div[a]) + om / p->eps + dpsi;","r[a] = p->eps * (dadphi + div[a]) + om / p->eps + dpsi;"),
 ("double tau = den != 0.0 ? num / den : tsum / (double)npair;","double tau = den != 0.0 ? num / den / 2 : tsum / (double)npair;"),
 ("c[i] = -s - B[i];","c[i] = -s + B[i];"),
 ("out[i] = -s - p->B1[a][i];","out[i] = s - p->B1[a][i];"),
 ("double dTdt = -p->G * p->v;","double dTdt = p->G * p->v;"),
 ("for (int d = 0; d < 3; ++d) dot += (ph[a] * g[b][d] - ph[b] * g[a][d]) * g[b][d];","for (int d = 0; d < 3; ++d) dot += (ph[a] * g[b][d] - ph[b] * g[a][d]) * g[a][d];"),
 ("if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue;","if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue; if (a==0) continue;"),
 ("dtp[a] = ((rd(o, F_PHI_DST, a, x, y, z) - vp) + (rd(o, F_PHI_DST, a, qx, qy, qz) - vq)) / (2.0 * p->dt);","dtp[a] = ((rd(o, F_PHI_DST, a, x, y, z) - vp) + (rd(o, F_PHI_DST, a, qx, qy, qz) - vq)) / (1.0 * p->dt);"),
]
try:
  for a,b in muts:
    assert orig.count(a)==1, a
    open(src,'w').write(orig.replace(a,b))
    r=subprocess.run([sys.executable,'-m','pytest','/root/repo/tests/test_oracle_pins.py','-q','-x','-p','no:cacheprovider'],capture_output=True,text=True,cwd='/root/repo')
    last=[l for l in r.stdout.splitlines() if 'passed' in l or 'failed' in l]
    fails=[l for l in r.stdout.splitlines() if l.startswith('FAILED')]
    print(('CAUGHT ' if r.returncode else 'MISSED ')+b[:60], fails[:1])
finally:
  open(src,'w').write(orig)

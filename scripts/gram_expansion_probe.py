import sys; sys.path.insert(0,'/root/repo')
import numpy as np
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma, uniform_pool
def ulp(x): return np.spacing(np.abs(x).astype(np.float32)).astype(np.float64)
def run(X, g, label):
    X32 = X.astype(np.float32); N = 2048; X32 = X32[:N]
    X64 = X32.astype(np.float64)
    d2_64 = ((X64[:,None,:]-X64[None,:,:])**2).sum(-1)
    K64 = np.exp(-g*d2_64)
    # direct form fp32 (sequential fma-like: fp32 ops)
    acc = np.zeros((N,N), np.float32)
    for k in range(X32.shape[1]):
        df = (X32[:,None,k]-X32[None,:,k]).astype(np.float32)
        acc = (acc + df*df).astype(np.float32)
    Kd = np.exp((-np.float32(g))*acc).astype(np.float32)
    # expansion, centered, dot in fp32 sequential (emulating TC fp32 accumulation)
    c = X32.mean(0).astype(np.float32)
    Xc = (X32 - c).astype(np.float32)
    nx = np.zeros(N, np.float32)
    for k in range(X32.shape[1]): nx = (nx + Xc[:,k]*Xc[:,k]).astype(np.float32)
    dot = np.zeros((N,N), np.float32)
    for k in range(X32.shape[1]): dot = (dot + (Xc[:,None,k]*Xc[None,:,k]).astype(np.float32)).astype(np.float32)
    d2e = ((nx[:,None]+nx[None,:]).astype(np.float32) - (np.float32(2)*dot)).astype(np.float32)
    d2e = np.maximum(d2e, 0)
    Ke = np.exp((-np.float32(g))*d2e).astype(np.float32)
    np.fill_diagonal(Ke, 1.0)
    bound = ulp(K64)*(1+g*d2_64)
    for name, K in (("direct", Kd), ("expansion-centered", Ke)):
        r = np.abs(K.astype(np.float64)-K64)/bound
        print(f"{label:10s} {name:20s} max {r.max():.2f} ulp*(1+g d2), p99.99 {np.quantile(r,0.9999):.2f}")
_, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 4096, 3); run(X, median_gamma(X,3), "knob16")
X = uniform_pool(4096, 16, 5); run(X, median_gamma(X,5), "uniform16")
X = uniform_pool(4096, 30, 5); run(X, median_gamma(X,5), "uniform30")

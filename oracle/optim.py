"""ORACLE (test infrastructure only) — the optimizer step OS (Table 3).

The paper names the instruction but not the optimizer; reading A27: AdamW as in
Loshchilov & Hutter (decoupled weight decay) with bias correction, fp32 master weights and fp32
moments, applied to every parameter with the same hyper-parameters. Written out plainly.
"""
import numpy as np


def adamw_step(params, grads, m, v, step, lr, beta1=0.9, beta2=0.95, eps=1e-8, weight_decay=0.1):
    """One AdamW update (step counts from 1). Updates params, m, v in place (dicts of arrays).
      m <- b1 m + (1-b1) g ;  v <- b2 v + (1-b2) g^2
      p <- p - lr * ( (m / (1-b1^t)) / (sqrt(v / (1-b2^t)) + eps) + wd * p )"""
    bc1 = 1.0 - beta1 ** step
    bc2 = 1.0 - beta2 ** step
    for k in params:
        g = grads[k]
        m[k] = beta1 * m[k] + (1.0 - beta1) * g
        v[k] = beta2 * v[k] + (1.0 - beta2) * g * g
        update = (m[k] / bc1) / (np.sqrt(v[k] / bc2) + eps) + weight_decay * params[k]
        params[k] = params[k] - lr * update
    return params, m, v

"""The paper's two prediction workflows, composed from the C-ABI calls
(SURVEY.md 8(f) NEXT-3 and NEXT-4).  Argument marshalling and selection only:
every numerical step runs in libbf.so kernels (bf_fit, bf_predict,
bf_oob_importance, bf_importance_finalize, bf_pca, bf_glm_gaussian,
bf_glm_predict, bf_mars_fit, bf_mars_predict, bf_rank_similarity); the host
picks rows and columns.

problem_scaling  -- P:173 ("we can use the models to generate values for the
    most influential variables from an unseen problem size for which the
    execution time will be predicted by the random forest"), P:222-224 (MM:
    80:20 split, keep the first 6-8 important variables, re-validate, model
    them as generalized linear models of the matrix size, predict unseen
    sizes), P:256 (NW: the same with MARS models, R earth).
hardware_scaling -- P:258-274 (machine characteristics of Table 2 injected
    as predictors; train on some GPUs, predict another), P:260/P:295 (the
    importance rankings of the platforms compared: "similarity").
"""
from __future__ import annotations


from . import (fit, glm_gaussian, glm_predict, importance_finalize, mars_fit, mars_predict, pca, pca_retained,
               prediction_error, rank_similarity)
from . import log_size_design as _log_size_design


def _torch():
    import torch
    return torch


def inc_mse(forest, X, y) -> "object":
    """%IncMSE of a forest's predictors (bf_oob_importance + bf_importance_finalize; S7)."""
    acc = forest.oob_importance(X, y)
    return importance_finalize(acc["d_slots"], acc["npur_slots"], acc["oob_sum"], acc["oob_cnt"], y)


def log_size_design(size) -> "object":
    """Default GLM design of one problem characteristic s (reading R26): [1, u, u^2, u^3], u = standardised
    log2 s (the paper's sizes span 2^5..2^11 and 64..8192), computed by bf_log_size_design.
    size: (n,) device tensor -> (4, n)."""
    return _log_size_design(size.contiguous())


def problem_scaling(X, y, size_row: int, train, test, top: int = 6, ntree: int = 500, seed: int = 0,
                    design=log_size_design, counter_model: str = "glm") -> dict:
    """X: (p, n) device tensor, y: (n,), size_row: the predictor holding the problem size, train/test: index
    tensors.  Returns the retained predictors, the re-validated forest's OOB statistics, the counter models
    (counter_model "glm": R26, P:224 for MM; "mars": R28, P:256 for NW), the modelled counters of the test
    rows and the predicted test times (MSE, explained variance)."""
    torch = _torch()
    Xtr, ytr = X[:, train].contiguous(), y[train].contiguous()
    f_all = fit(Xtr, ytr, ntree=ntree, seed=seed)
    imp = inc_mse(f_all, Xtr, ytr)
    f_all.free()
    order = torch.argsort(imp["inc_mse"], descending=True, stable=True)
    keep = order[:top].tolist()
    keep_c = [j for j in keep if j != size_row]                 # counters to model
    Xk = X[keep][:, train].contiguous()
    f_keep = fit(Xk, ytr, ntree=ntree, seed=seed + 1)           # re-validation on the retained set
    imp_k = inc_mse(f_keep, Xk, ytr)
    # counters as models of the problem size (GLM P:224 / MARS P:256), predicted for the test sizes
    Xh = torch.empty((len(keep), int(test.numel())), dtype=torch.float64, device=X.device)
    models = None
    if keep_c and counter_model == "mars":
        Str, Ste = X[size_row, train][None, :].contiguous(), X[size_row, test][None, :].contiguous()
        models = {"mars": [mars_fit(Str, X[j, train].contiguous()) for j in keep_c]}
        models["deviance"] = torch.tensor([m["rss"] for m in models["mars"]], dtype=torch.float64)
        models["null_deviance"] = None
        models["coef"] = None
        mod = torch.stack([mars_predict(m, Ste) for m in models["mars"]])
    elif keep_c:
        Ztr = design(X[size_row, train].contiguous())
        Zte = design(X[size_row, test].contiguous())
        models = glm_gaussian(Ztr, X[keep_c][:, train].contiguous())
        mod = glm_predict(Zte, models["coef"])
    if keep_c:
        for i, j in enumerate(keep):
            if j != size_row:
                Xh[i] = mod[keep_c.index(j)]
    for i, j in enumerate(keep):
        if j == size_row:
            Xh[i] = X[size_row, test]
    yh_sum, yh = f_keep.predict(Xh.contiguous(), ntree_total=ntree)
    yte = y[test].contiguous()
    mse, expl = prediction_error(yh.contiguous(), yte)
    f_keep.free()
    return {"keep": keep, "oob_mse": float(imp_k["oob_mse"]), "rsq": float(imp_k["rsq"]),
            "models": models, "deviance": None if models is None else models["deviance"],
            "null_deviance": None if models is None else models["null_deviance"],
            "coef": None if models is None else models["coef"], "X_model": Xh, "yhat": yh,
            "test_mse": mse, "test_explained": expl}


def n_components(sdev, frac: float = 0.97, cap: int = 10) -> int:
    """Reading R15: smallest k with cumulative variance >= frac, capped at 10 (P:134 '<10', P:189 '>97%');
    computed by bf_pca_retained on the device."""
    return pca_retained(sdev, frac, cap)


def hardware_scaling(counters, L, M, y, gen, train_gens=(0, 1), test_gen: int = 2, ntree: int = 500,
                     seed: int = 0) -> dict:
    """counters: (c, n) device tensor, L: (n,) problem size, M: (7, n) machine metrics (Table 2), y: (n,),
    gen: (n,) generation ids.  RF inputs = [PCA scores (k) | L | M]; train on train_gens, predict
    test_gen; similarity (R27) of the importance rankings of per-generation forests."""
    torch = _torch()
    pc = pca(counters.contiguous(), scale=True, k=None)
    k = n_components(pc["sdev"])
    R = torch.cat([pc["scores"][:k], L[None, :], M], dim=0).contiguous()
    tr = torch.nonzero(torch.isin(gen, torch.tensor(list(train_gens), device=gen.device))).flatten()
    te = torch.nonzero(gen == test_gen).flatten()
    Rtr, ytr = R[:, tr].contiguous(), y[tr].contiguous()
    f = fit(Rtr, ytr, ntree=ntree, seed=seed)
    imp = inc_mse(f, Rtr, ytr)
    _, yh = f.predict(R[:, te].contiguous(), ntree_total=ntree)
    f.free()
    yte = y[te].contiguous()
    mse, expl = prediction_error(yh.contiguous(), yte)
    per_gen = []
    for g in train_gens:
        ig = torch.nonzero(gen == g).flatten()
        Rg, yg = R[:, ig].contiguous(), y[ig].contiguous()
        fg = fit(Rg, yg, ntree=ntree, seed=seed + 1 + int(g))
        per_gen.append(inc_mse(fg, Rg, yg)["inc_mse"])
        fg.free()
    sims = {}
    for a in range(len(train_gens)):
        for b in range(a + 1, len(train_gens)):
            sims[(train_gens[a], train_gens[b])] = rank_similarity(per_gen[a], per_gen[b])
    return {"k": k, "inputs": R, "oob_mse": float(imp["oob_mse"]), "rsq": float(imp["rsq"]), "yhat": yh,
            "test_mse": mse, "test_explained": expl,
            "inc_mse_per_gen": per_gen, "similarity": sims}

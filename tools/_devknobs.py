"""Development tools only: map PM_* environment variables of the *tool's*
process onto explicit pm.tuning_set overrides (the library itself never reads
the environment).  PM_TRAP_V=3 -> tuning_set("trap_variant", 3), etc."""
import os

_MAP = {"PM_TRAP_V": "trap_variant", "PM_TRAP_W": "trap_W", "PM_TRAP_CLUSTER": "trap_cluster",
        "PM_TRAP_NBSYNC": "trap_nbsync", "PM_TRAP_CPC": "trap_cpc", "PM_TRAP_PROF": "trap_prof",
        "PM_TRAP_EP": "trap_ep", "PM_TRAP_VEC": "trap_vec", "PM_TRAP_SPEC": "trap_spec",
        "PM_TRAP_COAL": "trap_coal", "PM_SAD_PLAN": "sad_plan",
        "PM_TRAP_WAIT_MS": "trap_wait_ms", "PM_LS_SPARSE": "ls_sparse", "PM_LS_SPARSE_T": "ls_sparse_T",
        "PM_LS_CWALK": "ls_cwalk", "PM_LS_CWALK_C": "ls_cwalk_c", "PM_LS_SPARSE_GMEM": "ls_sparse_gmem", "PM_AUCTION_GS": "auction_gs",
        "PM_AUCTION_KEEP": "auction_keep", "PM_AUCTION_SMEM_PRICE": "auction_smem_price",
        "PM_AUCTION_THETA": "auction_theta", "PM_AUCTION_EPS_SHIFT": "auction_eps_shift",
        "PM_AUCTION_MAX_ROUNDS": "auction_max_rounds", "PM_AUCTION_CTAS_PER_SM": "auction_ctas_per_sm"}


def apply(pm):
    for env, name in _MAP.items():
        v = os.environ.get(env)
        if v not in (None, ""):
            pm.tuning_set(name, int(v))

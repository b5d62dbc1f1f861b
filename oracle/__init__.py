"""Oracle package -- TEST INFRASTRUCTURE ONLY (see emb_oracle.py header).

Importable only from tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs.  Never imported by paper_conf_sc_chenbyo24_b200.
"""
from .emb_oracle import *  # noqa: F401,F403
from .emb_oracle import __all__  # noqa: F401

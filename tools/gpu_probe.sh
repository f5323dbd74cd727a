#!/bin/bash
python - <<'PY'
import sys; sys.path.insert(0,'.')
import numpy as np, synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
for td in [(64,64,16),(64,32,16)]:
    d=T.Domain((128,64,64),td,ghost=2,two_step=1); d.load(synth.uniform_grid(128,64,64,1)); d.run(T.heat7(),4,2); d.sync()
    print(td, d.info["steps_per_pass"])
PY

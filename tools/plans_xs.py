import os, sys
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
for l in wl.RESNET50_F16 + wl.VGG16_F16:
    p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    os.environ["WINRS_FORCE_TA"]="2"
    try:
        q = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
        qs=(q.kernel_name, q.info['csplit'], q.info['Z'], round(q.model_us,1))
    except Exception as ex: qs=str(ex)
    del os.environ["WINRS_FORCE_TA"]
    print(l.name, p.kernel_name, p.info['csplit'], p.info['Z'], round(p.model_us,1), '|', qs)

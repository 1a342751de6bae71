#!/bin/bash
# compute-sanitizer on cfg1 (2-D, auto batches: the cooperative multi-batch launch with grid barriers), mini720 and mini3d
#!/bin/bash
timeout 600 python -m pytest tests/test_gpu_slabs.py -x -q > gpurun_out/s3san_slabs.log 2>&1; echo "rc=$?" >> gpurun_out/s3san_slabs.log
cat > /tmp/san_case.py <<'PY'
import sys, numpy as np
sys.path.insert(0, '.')
import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import CONFIGS, WorkloadConfig, make_case
for cfg, nb, q in ((CONFIGS["cfg1"], 8, 1), (WorkloadConfig("mini720", 48, 2, 720, 96, 9, 26, 0.005), 26, 1), (WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002), 26, 0)):
    case = make_case(cfg)
    g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    for det in (0, 1):
        with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=nb), M.Options(sv_side=cfg.sv_side, deterministic=det, quantize_A=q)) as r:
            r.set_sinogram(case.y, case.w)
            r.init_fbp()
            r.iterate(3)
            r.set_update_dump(100000); r.iterate(1); r.update_dump(10)
            print(cfg.name, det, float(r.image().max()))
PY
for tool in memcheck racecheck synccheck initcheck; do
  timeout 500 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san_case.py > gpurun_out/s3san_$tool.log 2>&1; echo "rc=$?" >> gpurun_out/s3san_$tool.log
done

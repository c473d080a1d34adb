# build-time tile selection (autotune) A/B via ARLO_NO_AUTOTUNE; tests; tiles chosen
mkdir -p gpurun_out/ab29
python __graft_entry__.py > gpurun_out/ab29/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_runtime.py -q -m gpu -k "autotuned or tiny or cross_length" > gpurun_out/ab29/rt_tests.log 2>&1; echo RC=$? >> gpurun_out/ab29/rt_tests.log
for rep in 1 2; do
  python tools/ab_forward.py | sed "s/^/tuned /"
  ARLO_NO_AUTOTUNE=1 python tools/ab_forward.py | sed "s/^/plain /"
done > gpurun_out/ab29/fwd.txt 2>&1
python - > gpurun_out/ab29/tiles.txt 2>&1 <<'PY'
import torch, sys
sys.path.insert(0, '.')
from paper_conf_icpp_tanlyl024_b200 import arlo, workload as wl
for name, cfg, Ls, mb in (("base", wl.BERT_BASE, (64, 128, 256, 512), 32), ("large", wl.BERT_LARGE, (256, 512), 64)):
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16, torch.device("cuda")), arlo.BF16)
    for L in Ls:
        rt = arlo.Runtime(W, L, mb)
        print(name, L, {n: rt.gemm_tiles(n) for n in (1, 8, 16, 32, mb)}, flush=True)
        rt.close()
PY
timeout 900 python bench.py > gpurun_out/ab29/bench.json 2> gpurun_out/ab29/bench.err

# fused peer pushes (edge tiles' and band's stores into the neighbours) vs copy-engine pushes,
# multi-process on the box's GPU, plus the full GPU suite for the new kernel instantiations
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
for f in 1 0; do FFTSTENCIL_PEER_FUSED=$f timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node=3 --master-addr=127.0.0.1 --master-port=2953$f tests/_peer_worker.py 2>&1 | grep -E "case|Error|error" | head -8; done
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -3
ENV_AB_ROUNDS=1 timeout 600 python tools/env_ab.py heat3d heat2d 2>&1 | grep device

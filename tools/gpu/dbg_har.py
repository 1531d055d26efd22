import numpy as np, torch, sys
sys.path.insert(0, '.')
import oracle, synth
import paper_conf_ipps_qiaoth21_b200 as isp
oracle.build_oracle()
for (h, w) in [(70, 2064), (33, 4112), (8, 8), (40, 256), (40, 512)]:
    img = synth.structured_u8(h, w, 11)
    for mode in ["clamp", "mirror", "repeat", "constant"]:
        rdx, rdy, _ = oracle.sobel(img, mode, 45)
        ref = oracle.harris(rdx, rdy, mode, -3, 0)
        got = isp.isp_harris_u8(torch.from_numpy(rdx).cuda(), torch.from_numpy(rdy).cuda(), mode, -3, 0, variant="tma").cpu().numpy()
        bad = np.argwhere(got != ref)
        print(h, w, mode, len(bad), isp.isp_last_plan()["tile_h"], "rows", sorted(set(bad[:, 0].tolist()))[:20], "cols", sorted(set((bad[:, 1] % 128).tolist()))[:20], "strips", sorted(set((bad[:, 1] // 128).tolist()))[:10])

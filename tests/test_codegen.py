"""CPU check of the query compiler: libhq generates the fused kernel's CUDA
source for a matrix of pipeline shapes (staged / global compact / direct /
linear probes; scalar, dense, lane-private, shared-hash and global-hash
group-by sinks; materialisation; the C2 atomic ablation; R=2 and R=4) and every
source must compile with NVRTC for sm_100a.  No GPU is needed (NVRTC is a
compiler); the fake device pointers are never dereferenced."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sigmod_funkebnmt18_b200")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


@pytest.fixture(scope="module")
def checker(tmp_path_factory):
    from paper_conf_sigmod_funkebnmt18_b200 import build
    build.build()
    if not os.path.exists(NVCC):
        pytest.skip("nvcc not available")
    exe = str(tmp_path_factory.mktemp("codegen") / "jit_codegen_check")
    cmd = [NVCC, "-O1", "-std=c++17", "-I" + os.path.join(ROOT, "include"), "-I" + os.path.join(PKG, "csrc"),
           os.path.join(ROOT, "tests", "codegen", "jit_codegen_check.cu"), "-o", exe, "-L" + PKG, "-lhq", "-lnvrtc",
           "-Xlinker", "-rpath", "-Xlinker", PKG, "-Xlinker", "-rpath", "-Xlinker", "/usr/local/cuda/lib64"]
    subprocess.run(cmd, check=True, capture_output=True)
    return exe


def test_generated_kernels_compile(checker, tmp_path):
    env = {k: v for k, v in os.environ.items() if not k.startswith("HQ_")}
    p = subprocess.run([checker, str(tmp_path)], capture_output=True, text=True, env=env, timeout=600)
    assert p.returncode == 0, p.stdout + p.stderr
    assert p.stdout.startswith("OK 32 of 32"), p.stdout
    srcs = {f[:-3]: open(tmp_path / f).read() for f in os.listdir(tmp_path)}
    # the probe kinds the shapes were built to exercise are present
    rk = srcs["ranked_probes"]  # ranked sparse-key tables: {bits, dir} pair, popcount, payload row
    assert "__ldg((const uint2*)p.pf[0] + (e_[r] >> 5))" in rk and "k_[r] + __popc(w_[r]" in rk
    assert "(const int2*)p.rpay[0] + rk_" in rk and "__ldg(p.rpay[2] + rk_)" in rk
    assert "__ldg(p.pf[1] + (e_[r] >> 5)) : 0u" in rk and "p.rpay[1]" not in rk  # semi-join: bits only
    assert "p.ht[0]" not in rk and "0x9E3779B1u" not in rk.split("gk_")[0]
    # the shared-memory request of a kernel whose probes read global memory stays inside the
    # 196-KB carve-out (60 KB of L1 for those probes; hq_plan.cu layout search)
    def defs(src):
        out = {}
        for line in src.splitlines():
            if line.startswith("#define ") and len(line.split()) == 3:
                _, k, v = line.split()
                out[k] = v.rstrip("u")
        return out
    for name in ("star_dense_lrgp", "ranked_probes", "global_hash_groups"):
        d = defs(srcs[name])
        request = int(d["OFF_STAGE"]) + int(d["S"]) * int(d["STAGE_STRIDE"])
        assert request <= 196 * 1024 - 1024 and int(d["S"]) >= 3, (name, request, d["S"], d["NW"])
    # the warp update queue of a global hash group table keeps the ring's stages
    assert int(defs(srcs["global_hash_groups"])["GQ_CAP"]) >= 4
    star = srcs["star_dense_lrgp"]
    assert "lds_u32(sm0_ + " in star                 # staged bitmap
    assert "__ldg((const unsigned char*)p.ctab[" in star  # global byte map
    assert "__ldg((const u32*)p.ctab[" in star       # global bitmap
    assert "& 15u" in star                           # staged nibbles
    assert "mbar_wait_sleep" in star
    assert "__ldg((const int4*)p.ht[" in srcs["materialise_lrgp"]  # 4-word direct slots
    assert "p.pf[" in srcs["materialise_lrgp"]                     # linear prefilter
    # global hash groups behind no shared table: warp update queues (gq_flush) at R = 2,
    # warp compaction at R = 4
    assert "gq_flush(p, sagg, sl0_, gq_, gqn_)" in srcs["global_hash_groups"] and "pre_[R]" in srcs["global_hash_groups_r4"]
    assert "#define GQ_CAP 0u" in srcs["global_hash_groups_r4"]
    # group keys narrowed to the build-side payload ranges: dense shared table + key remap at the merge
    assert "software-pipelined" not in star  # opt-in only (HQ_JIT_SWP=1)
    assert "#define SMODE 0" in srcs["star_smem_hash"]  # dense domain larger than any shared table: global (C2 + warp merging)
    narrowed = srcs["star_narrowed_dense"]
    assert "#define SMODE 1" in narrowed and "#define SMEM_CAP 1183u" in narrowed and "gkey_ +=" in narrowed
    # ... and by the rank among the payloads' distinct values (5 of the 21 codes 4..24)
    ranked = srcs["star_ranked_dense"]
    assert "#define SMEM_CAP 175u" in ranked and "dv_[o_]" in ranked
    # rank-coded byte maps: the probe stores the rank, the group index uses it directly,
    # and RV_ maps it back to the value where the value is needed
    assert "RV_0[256] = {4, 9, 10, 13, 24}" in ranked and "__popc(0x00100261u" not in ranked
    # multi-pass (A1/B1/C1): the count kernel writes flags and skips the sink;
    # the write kernel reads flags + positions, skips filters / semi probes
    c1 = srcs["star_ranked_dense_mp1"]
    assert "fl_[row_] = " in c1 and "group_update(" not in c1.split("extern \"C\"")[1]
    w2 = srcs["materialise_lrgp_mp2"]
    assert "pos_ = (u64)(u32)" in w2 and "atomicAdd(p.counter" not in w2 and "(int)c4" not in w2
    assert "((u64*)p.out[0])[pos_] = gk_[r];" in srcs["star_ranked_dense_mp2"]
    # high-cardinality hash group-by skips the shared table (C2 straight to global)
    assert "#define SMODE 0" in srcs["global_hash_groups"]
    # LEFT OUTER probes keep the row and default the payload to 0; predicate instructions
    op = srcs["outer_predicates"]
    assert "[R] = {};" in op and "(void)f_" in op
    assert "= RV_0[b_ & 255u];" in op  # a rank-coded byte map decoded at an OUTER probe
    assert "(a_ != 0 && " in op and "3855ULL >> v_" in op and "(a_ != 0 || " in op
    assert "(void)f_" not in srcs["outer_predicates_mp2"].split("extern \"C\"")[0]
    # composite keys: the slot's word 1 is compared with the second key, payloads start at word 2
    cp = srcs["composite_probe"]
    assert "kk2_[r] = (int)(long long)c2[r];" in cp and "sl_[r].y == kk2_[r]" in cp and "= sl_[r].z;" in cp

import os, sys
sys.path.insert(0, os.getcwd())
import paper_conf_icpp_liuwc21_b200 as fp
for env in [{}, {"PSO_CTAS": "1"}]:
    os.environ.pop("PSO_CTAS", None); os.environ.update(env)
    for n, d in ((64, 65536), (4096, 65536)):
        try:
            s = fp.Swarm(n, d, 0.9, 2, 2, -5.12, 5.12, 2, 1, device=0)
            i = s.info(); print(env, n, d, "ok cluster", i["cluster"], "stages", i["pipeline_stages"], "grid", i["grid"], "smem", i["smem_bytes"]); s.close()
        except Exception as e:
            print(env, n, d, "FAIL", e)

"""Debug aid: per-rank iterations / tail iterations / bodies / barrier arrivals of tests.test_gpu_mp.case_parity."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    from tests import mp_harness

    for world, part, kw in ((2, "random", {}), (2, "random", {})):
        res = mp_harness.run("tests.test_gpu_mp", "case_parity", world=world, args=(12, part, kw), timeout=300,
                             hide_gpu=False)
        for alg in res[0]:
            print(world, alg, [(r[alg]["iters"], r[alg]["tail_iters"], r[alg]["bodies"], r[alg]["osteal_iter"],
                                r[alg]["barriers"], r[alg]["last"]) for r in res], flush=True)


if __name__ == "__main__":
    main()

"""Pool geometries used by the pooling pins and parity tests: every (k, s, p, ceil) the
five networks use plus ragged/odd variants."""
GEOMS = [
    (2, 2, 2, 2, 0, 0, 0),  # VGG16 / OverFeat
    (3, 3, 2, 2, 0, 0, 0),  # AlexNet (floor)
    (3, 3, 2, 2, 0, 0, 1),  # NiN / GoogLeNet (ceil)
    (3, 3, 1, 1, 1, 1, 0),  # GoogLeNet in-module
    (2, 2, 2, 2, 0, 0, 1),
    (3, 3, 3, 3, 0, 0, 0),
    (3, 3, 2, 2, 1, 1, 0),
    (3, 3, 2, 2, 1, 1, 1),
    (2, 2, 1, 1, 0, 0, 0),
    (4, 4, 4, 4, 0, 0, 0),
    (2, 3, 2, 1, 1, 1, 0),
    (1, 1, 1, 1, 0, 0, 0),
]


def gid(g):
    return "k{}x{}s{}x{}p{}x{}{}".format(*g[:6], "c" if g[6] else "")

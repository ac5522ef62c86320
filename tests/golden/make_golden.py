"""Writes the small real-graph fixtures under tests/golden/ from networkx's
bundled copies (no oracle, no CUDA path involved).  Each file is a plain
"a b" edge list; the header names the source and the published triangle
count where one exists.

  karate.txt      Zachary's karate club (J. Anthropol. Res. 33, 1977):
                  34 vertices, 78 edges, 45 triangles (the count BASELINE.json's
                  north_star names as an oracle pin).
  lesmis.txt      Les Miserables co-appearance (Knuth, Stanford GraphBase):
                  77 vertices, 254 edges (T pinned by brute force in the test).
  florentine.txt  Florentine families (Padgett & Ansell 1993): 15 / 20.
  davis.txt       Davis southern women (bipartite, 1941): 32 / 89 -> T = 0.

Weights are dropped (SURVEY.md §4.2 pitfall: networkx karate carries weights).
"""
import os
import networkx as nx

HERE = os.path.dirname(os.path.abspath(__file__))


def write(name, G, note):
    nodes = {v: i for i, v in enumerate(G.nodes())}
    with open(os.path.join(HERE, name), "w") as f:
        f.write(f"# {note}\n# n={G.number_of_nodes()} m={G.number_of_edges()}\n")
        for a, b in G.edges():
            f.write(f"{nodes[a]} {nodes[b]}\n")


write("karate.txt", nx.karate_club_graph(), "Zachary karate club (1977); published T = 45")
write("lesmis.txt", nx.les_miserables_graph(), "Les Miserables co-appearance (Knuth SGB)")
write("florentine.txt", nx.florentine_families_graph(), "Florentine families (Padgett & Ansell 1993)")
write("davis.txt", nx.davis_southern_women_graph(), "Davis southern women, bipartite (1941); T = 0")
